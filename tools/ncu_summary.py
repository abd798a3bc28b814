"""Summarise ncu --set full captures (gpurun_out/prof_*.ncu-rep) into profiles/ncu_summary.json.

Run here (no GPU needed):  python tools/ncu_summary.py gpurun_out profiles/ncu_summary.json r01
Per kernel: duration, DRAM bytes (read + write) per launch, shared-memory wavefronts per request
for loads and stores, bank conflicts, issue-slot utilisation, occupancy, registers.
"""
import csv
import io
import json
import os
import subprocess
import sys

CAPTURES = {
    "transpose_b32_rap": "prof_t32_rap", "transpose_b32_raw": "prof_t32_raw",
    "transpose_b32_pad": "prof_t32_pad", "transpose_b32_xor": "prof_t32_xor",
    "transpose_b32_ras": "prof_t32_ras", "transpose_b64_rap": "prof_t64_rap",
    "transpose_b64_rap16": "prof_t64_rap16", "transpose_b64_rap64": "prof_t64_rap64",
    "sweep_w32": "prof_sweep", "sweep_w32_match": "prof_sweep_match", "trace_w32": "prof_trace",
}

# work units per captured launch (tools/gpu_profile.sh command lines)
UNITS = {"sweep_w32": ("trials", 8388608), "sweep_w32_match": ("trials", 4194304),
         "trace_w32": ("evaluations", 4096 * 2048 * 5),
         "transpose_b32_rap": ("bytes", 2 * 8192 * 8192 * 4), "transpose_b32_raw": ("bytes", 2 * 8192 * 8192 * 4),
         "transpose_b32_pad": ("bytes", 2 * 8192 * 8192 * 4), "transpose_b32_xor": ("bytes", 2 * 8192 * 8192 * 4),
         "transpose_b32_ras": ("bytes", 2 * 8192 * 8192 * 4), "transpose_b64_rap": ("bytes", 2 * 16384 * 16384 * 8),
         "transpose_b64_rap16": ("bytes", 2 * 16384 * 16384 * 8),
         "transpose_b64_rap64": ("bytes", 2 * 16384 * 16384 * 8)}

WANT = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum",
        "smsp__sass_inst_executed_op_shared_ld.sum", "smsp__sass_inst_executed_op_shared_st.sum",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum",
        "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__inst_executed.sum",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active", "sm__cycles_active.avg"]

# ALU pipe (LOP3 / SHF / ISETP / IADD3 / PRMT ...): reciprocal throughput 2 cycles per warp
# instruction per SMSP (B300_MICROARCH.md "Pipe rates"), i.e. 2 warp-instructions / clk / SM
ALU_WARP_INST_PER_SM_CLK = 2.0
N_SMS = 148

SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-9, "us": 1e-6, "ms": 1e-3,
         "nsecond": 1e-9, "usecond": 1e-6,
         "msecond": 1e-3, "second": 1.0}


def _page(rep, page):
    """ncu's CSV export of a capture: <stem>.<page>.csv written on the GPU box (tools/ncu_export.sh),
    else ncu -i on the .ncu-rep here."""
    stem = rep[:-len(".ncu-rep")] if rep.endswith(".ncu-rep") else rep
    csv_path = f"{stem}.{page}.csv"
    if os.path.exists(csv_path):
        return open(csv_path).read()
    if os.path.exists(csv_path + ".gz"):
        import gzip
        return gzip.open(csv_path + ".gz", "rt").read()
    args = ["ncu", "-i", rep, "--page", page, "--csv"] + (["--print-source", "sass"] if page == "source" else [])
    return subprocess.run(args, capture_output=True, text=True).stdout


def raw_metrics(rep):
    out = _page(rep, "raw")
    rows = list(csv.reader(io.StringIO(out)))
    head, units, vals = rows[0], rows[1], rows[2]
    d = {}
    for h, u, v in zip(head, units, vals):
        if h in WANT:
            try:
                x = float(v.replace(",", ""))
            except ValueError:
                continue
            d[h] = x * SCALE.get(u, 1.0)
    d["kernel_name"] = vals[head.index("Kernel Name")] if "Kernel Name" in head else None
    return d


def source_smem(rep):
    """Per-instruction shared-memory wavefronts from the source page: (ld_wf, ld_inst, st_wf, st_inst, excessive)."""
    out = _page(rep, "source")
    rows = list(csv.reader(io.StringIO(out)))
    if len(rows) < 3:
        return None
    head = rows[1]
    acc = [0.0] * 5
    for r in rows[2:]:
        if len(r) != len(head):
            continue
        d = dict(zip(head, r))
        src = d.get("Source", "")
        op = src.split()[0] if src.split() else ""
        if op.startswith("@"):
            op = src.split()[1]
        try:
            wf = float(d.get("L1 Wavefronts Shared") or 0)
            n = float(d.get("Instructions Executed") or 0)
            ex = float(d.get("L1 Wavefronts Shared Excessive") or 0)
        except ValueError:
            continue
        if op.startswith("LDS"):
            acc[0] += wf; acc[1] += n
        elif op.startswith("STS"):
            acc[2] += wf; acc[3] += n
        acc[4] += ex
    return acc


def main(src_dir, dst, tag):
    kernels = {}
    for key, stem in CAPTURES.items():
        rep = None
        for cand in (stem, f"{tag}_{stem}"):            # committed copies: profiles/<tag>_<stem>
            base = os.path.join(src_dir, cand)
            if os.path.exists(base + ".ncu-rep") or os.path.exists(base + ".raw.csv"):
                rep = base + ".ncu-rep"
                break
        if rep is None:
            continue
        m = raw_metrics(rep)
        ld_w = m.get("l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum")
        st_w = m.get("l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum")
        ld_i = m.get("smsp__sass_inst_executed_op_shared_ld.sum")
        st_i = m.get("smsp__sass_inst_executed_op_shared_st.sum")
        dram = (m.get("dram__bytes_read.sum") or 0) + (m.get("dram__bytes_write.sum") or 0)
        kernels[key] = {
            "source": f"profiles/{tag}_{stem}.ncu-rep[.gz] / .raw.csv / .source.csv (ncu --set full --clock-control none)",
            "kernel_name": m.get("kernel_name"),
            "duration_us_cold": m.get("gpu__time_duration.sum", 0) * 1e6,
            "dram_bytes_read": m.get("dram__bytes_read.sum"), "dram_bytes_write": m.get("dram__bytes_write.sum"),
            "dram_bytes_per_launch": dram or None,
            "dram_throughput_pct": m.get("dram__throughput.avg.pct_of_peak_sustained_elapsed"),
            "smem_wavefronts_per_request": {"ld": ld_w / ld_i if ld_i else None,
                                            "st": st_w / st_i if st_i else None},
            "smem_bank_conflicts": {"ld": m.get("l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum"),
                                    "st": m.get("l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum")},
            "issue_active_frac": (m.get("smsp__issue_active.avg.pct_of_peak_sustained_active") or 0) / 100,
            "warps_active_pct": m.get("sm__warps_active.avg.pct_of_peak_sustained_active"),
            "registers": m.get("launch__registers_per_thread"), "grid": m.get("launch__grid_size"),
            "block": m.get("launch__block_size"), "instructions": m.get("smsp__inst_executed.sum"),
        }
        sm = source_smem(rep)
        if sm:
            kernels[key]["smem_wavefronts_per_request"] = {"ld": sm[0] / sm[1] if sm[1] else None,
                                                           "st": sm[2] / sm[3] if sm[3] else None}
            kernels[key]["smem_wavefronts_excessive"] = sm[4]
            kernels[key]["smem_wavefronts_note"] = ("per-instruction L1 Wavefronts Shared / executed LDS|STS "
                                                    "(source page); l1tex__data_bank_conflicts also counts "
                                                    "inter-instruction arbitration")
        if key in UNITS:
            unit, n = UNITS[key]
            kernels[key]["units_per_launch"] = {unit: n}
            if m.get("smsp__inst_executed.sum"):
                kernels[key][f"warp_instructions_per_{unit[:-1]}"] = m["smsp__inst_executed.sum"] / n
            alu_pct = m.get("sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active")
            cyc = m.get("sm__cycles_active.avg")
            if alu_pct is not None and cyc:
                alu = alu_pct / 100 * ALU_WARP_INST_PER_SM_CLK * N_SMS * cyc
                kernels[key]["alu_pipe_active_frac"] = alu_pct / 100
                kernels[key][f"alu_warp_instructions_per_{unit[:-1]}"] = alu / n
    # steady-state DRAM traffic (ncu --cache-control none, consecutive launches): the dirty lines
    # a launch leaves in L2 are written back during the next one, so per-launch read + write
    # bytes here are the true cost (the --set full captures flush caches between replays)
    for key, stem in (("transpose_b32_rap", "steady_t32"), ("transpose_b64_rap", "steady_t64"),
                       ("transpose_b64_rap16", "steady_t64_rap16"), ("transpose_b64_rap64", "steady_t64_rap64")):
        path = os.path.join(src_dir, stem + ".csv")
        if not os.path.exists(path):
            path = os.path.join(src_dir, f"{tag}_steady_dram_{stem[7:]}.csv")
        if key not in kernels or not os.path.exists(path):
            continue
        txt = open(path).read()
        txt = txt[txt.index('"ID"'):]
        per = {}
        for r in csv.DictReader(io.StringIO(txt)):
            if r["Metric Name"].startswith("dram__bytes"):
                per[r["ID"]] = per.get(r["ID"], 0.0) + float(r["Metric Value"].replace(",", "")) * SCALE.get(r["Metric Unit"], 1)
        if per:
            kernels[key]["dram_bytes_per_launch_steady"] = sum(per.values()) / len(per)
            kernels[key]["dram_steady_source"] = f"profiles/{tag}_steady_dram_{stem[7:]}.csv (--cache-control none)"
    os.makedirs(os.path.dirname(dst), exist_ok=True)
    json.dump({"round": tag, "note": "cold-cache, serialised ncu replays: compare shares and ratios, "
                                     "not absolute times; dram bytes exclude lines still dirty in L2 at exit",
               "kernels": kernels}, open(dst, "w"), indent=1)
    for k, v in kernels.items():
        print(f"{k:20s} {v['duration_us_cold']:8.1f} us  dram {v['dram_bytes_per_launch'] or 0:.3e} B  "
              f"smem wf/req ld {v['smem_wavefronts_per_request']['ld']} st {v['smem_wavefronts_per_request']['st']}  "
              f"issue {v['issue_active_frac']:.3f} regs {v['registers']}")


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "gpurun_out",
         sys.argv[2] if len(sys.argv) > 2 else "profiles/ncu_summary.json",
         sys.argv[3] if len(sys.argv) > 3 else "r01")
