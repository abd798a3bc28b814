"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv) into per-kernel shares."""
import csv
import io
import sys
from collections import defaultdict


def short(name):
    for key in ("transpose_kernel", "sweep_match_kernel", "sweep_kernel", "unpack_blocks", "trace_kernel",
                "congestion_kernel", "perm_gen_kernel"):
        if key in name:
            return "rapk::" + key + (name[name.index("<"):name.index(">") + 1] if "<" in name else "")
    return name.split("(")[0][:60]


def main(path):
    txt = open(path).read()
    txt = txt[txt.index('"ID"'):]
    agg = defaultdict(list)
    for r in csv.DictReader(io.StringIO(txt)):
        v = float(r["Metric Value"]) * {"ns": 1e-3, "us": 1.0, "ms": 1e3}.get(r["Metric Unit"], 1e-3)
        agg[short(r["Kernel Name"])].append(v)
    tot = sum(sum(v) for v in agg.values())
    print(f"{'kernel':60s} {'launches':>8s} {'mean us':>10s} {'share':>7s}")
    for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
        print(f"{k:60s} {len(v):8d} {sum(v) / len(v):10.1f} {sum(v) / tot * 100:6.1f}%")


if __name__ == "__main__":
    main(sys.argv[1])
