"""Commit-ready SASS of the default kernel instantiations (no GPU needed):
    python tools/sass_listings.py [librap.so] [profiles/sass]
Writes one listing per kernel (cuobjdump -sass) plus an opcode histogram, so the instruction mix
the DESIGN cites (LDG.E.128.CONSTANT / STS / LDS / STG, PREEXIT / ACQBULK for programmatic
dependent launch, UCGABAR cluster barriers, R2P + VOTE ballots, CREDUX, MATCH) can be checked."""
import collections
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KERNELS = {
    "transpose_b32_rap_cluster": "_ZN4rapk16transpose_kernelILi4ELi1ELb1ELi1ELi2ELb0ELi4ELi2ELb0ELb0ELi8ELb0EEEvPKjPjllllNS_10TileShiftsEjjbNS_7PeerOutE14CUtensorMap_st",
    "transpose_b64_rap_two_planes": "_ZN4rapk16transpose_kernelILi4ELi2ELb1ELi1ELi1ELb0ELi12ELi1ELb0ELb0ELi1ELb0EEEvPKjPjllllNS_10TileShiftsEjjbNS_7PeerOutE14CUtensorMap_st",
    "transpose_b64_rap64_slots": "_ZN4rapk18transpose64_kernelILi4ELb1ELi12ELi1ELb1EEEvPK5uint2PS1_llllNS_10TileShiftsEjj",
    "transpose_b64_rap16": "_ZN4rapk22transpose_rap16_kernelILi12EEEvPK5uint2PS1_llllNS_10TileShiftsEjj",
    "sweep32_w32_5pat_3sch": "_ZN4rapk14sweep32_kernelILj31ELj7EEEvjjjmmmPm",
    "trace32_w32_5sch": "_ZN4rapk14trace32_kernelILi32ELj31EEEvjmPKjmmmPm",
}


def main(lib, out_dir):
    os.makedirs(out_dir, exist_ok=True)
    summary = []
    for name, fn in KERNELS.items():
        txt = subprocess.run(["cuobjdump", "-sass", "-fun", fn, lib], capture_output=True, text=True).stdout
        ops = collections.Counter()
        for ln in txt.splitlines():
            m = re.match(r"\s+/\*[0-9a-f]+\*/\s+(.*?);", ln)
            if m:
                op = re.sub(r"^@!?U?P[0-9T] ", "", m.group(1)).split()[0]
                ops[op] += 1
        if not ops:
            sys.exit(f"{name}: no SASS for {fn} in {lib} (template signature changed?)")
        with open(os.path.join(out_dir, f"{name}.sass"), "w") as f:
            f.write(f"// cuobjdump -sass -fun {fn} {os.path.relpath(lib, ROOT)}\n")
            f.write("// opcode histogram (static): " + ", ".join(f"{k} {v}" for k, v in ops.most_common()) + "\n")
            f.write(txt)
        summary.append(f"{name}: {sum(ops.values())} instructions; " +
                       ", ".join(f"{k} {v}" for k, v in ops.most_common(14)))
    open(os.path.join(out_dir, "README.txt"), "w").write(
        "Static SASS of the default instantiations (tools/sass_listings.py):\n" + "\n".join(summary) + "\n")
    print("\n".join(summary))


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "paper_conf_icppw_nakanomi14_b200", "librap.so"),
         sys.argv[2] if len(sys.argv) > 2 else os.path.join(ROOT, "profiles", "sass"))
