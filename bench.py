"""bench.py -- RAP hot path on B200: one JSON line per run (driver contract).

A step is one pass of the whole hot path over one batch of synthetic input:
  T0-T3  RAP transpose of the BASELINE cfg3 matrix (8192 x 8192 float32, out-of-place,
         inputs 256 MiB > 126 MB L2, so no flush is needed between steps), and
  C1-C4  one batch of the cfg2 congestion sweep (w = 32, all 5 patterns x RAW/RAS/RAP;
         --sweep-trials per step, counter-based so batches are disjoint trial ranges).
`value` is the headline transpose throughput in GB/s: algorithmic bytes (read once + write
once) / the transpose kernels' device time inside the timed steps (CUDA events on the
launching stream).  The sweep is reported beside it as trials/s (`sweep`).

--workload picks another config as the timed step: sweep (cfg2 only), cfg4 (16384^2
float64), tile (cfg1 32x32), layouts (cfg3 under raw/pad/xor/ras/rap), dist (cfg5,
row-block-sharded 32768^2 with NCCL all-to-all; needs torchrun).
--impl reference times the CPU oracle (the only reference this paper has) on a bounded
sample of the same workload, on the host cores.

N > 1 (torchrun): every rank transposes its own cfg3 matrix (replicas; weak scaling) and
sweeps a disjoint trial range; the histograms are all-reduced over NCCL once per step.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "RAP transpose GB/s vs HBM peak; smem wavefronts/request; congestion trials/s"
ALL_PAT = ["contiguous", "stride", "diagonal", "random", "malicious"]
SCH = ["raw", "ras", "rap"]


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=50)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--impl", default="mine", choices=["mine", "reference"])
    p.add_argument("--workload", default="default",
                   choices=["default", "sweep", "cfg4", "tile", "layouts", "dist"])
    p.add_argument("--sweep-trials", type=int, default=1 << 24)
    p.add_argument("--layout", default="rap")
    p.add_argument("--sweep-algo", default="default", choices=["default", "match"])
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-cpu", action="store_true")
    return p.parse_args()


def load_peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(path):
        d = json.load(open(path))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, torch copy_)"
    return 6650.0, "fallback (B200_PROFILING.md: 6.65 TB/s)"


def load_traffic(kernel_key: str):
    """dram bytes per launch from the committed ncu --set full summary, if present."""
    path = os.path.join(ROOT, "profiles", "ncu_summary.json")
    if not os.path.exists(path):
        return None
    d = json.load(open(path))
    k = d.get("kernels", {}).get(kernel_key)
    return None if k is None else k.get("dram_bytes_per_launch")


class Clocks:
    """nvidia-smi sampler running during the timed region."""

    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "50"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except OSError:
            self.proc = None
        time.sleep(0.15)
        return self

    def __exit__(self, *a):
        if self.proc is None:
            self.result = {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
            return
        time.sleep(0.1)
        self.proc.terminate()
        out, _ = self.proc.communicate(timeout=10)
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in out.strip().splitlines():
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 7:
                continue
            try:
                sm.append(float(f[0]))
                mx.append(float(f[1]))
            except ValueError:
                continue
            for n, v in zip(names, f[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        self.result = {"sm_mhz": statistics.median(sm) if sm else None,
                       "sm_max_mhz": max(mx) if mx else None, "reasons": sorted(reasons),
                       "samples": len(sm)}


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


# ---------------------------------------------------------------------------- reference arm
def run_reference(args):
    """The CPU oracle timed on the host cores on a bounded sample of the workload."""
    ws, rank, _ = dist_env()
    if ws > 1 and rank != 0:
        return
    import numpy as np
    import torch

    import oracle
    import workloads
    threads = oracle.max_threads()
    if args.workload == "sweep":
        n = 20000
        unit, what = "trials/s", f"{n} trials of the w=32 sweep (5 patterns x RAW/RAS/RAP) per step"
        fn = lambda k: oracle.sweep(32, ALL_PAT, SCH, 1, k * n, n, threads=threads)
        work = n
    else:
        rows, cols, dt = (16384, 16384, torch.float64) if args.workload == "cfg4" else (8192, 8192, torch.float32)
        band = 512
        x = workloads.as_bits_numpy(workloads.random_bits(band, cols, dt, seed=0))
        unit = "GB/s"
        what = f"{band} x {cols} row band of the {rows}x{cols} {dt} matrix per step (oracle naive transpose)"
        fn = lambda k: oracle.transpose(x, threads=threads)
        work = 2 * x.nbytes / 1e9
    for k in range(args.warmup):
        fn(k)
    t0 = time.perf_counter()
    for k in range(args.steps):
        fn(args.warmup + k)
    dt_s = time.perf_counter() - t0
    value = work * args.steps / dt_s
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": unit, "n_gpus": ws,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt_s / args.steps * 1e3,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32",
            "data": "synthetic",
            "config": {"workload": args.workload if args.workload != "default" else "cfg3 8192x8192 float32 transpose"},
            "cpu_baseline": {"value": value, "unit": unit, "cores": threads, "kind": "oracle", "sample": what},
            "e2e": {"value": value, "unit": unit, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------------------- our arm
def cpu_baseline_transpose(rows, cols, dt):
    import oracle
    import workloads
    threads = oracle.max_threads()
    band = 1024
    x = workloads.as_bits_numpy(workloads.random_bits(band, cols, dt, seed=0))
    oracle.transpose(x, threads=threads)
    reps, t0 = 0, time.perf_counter()
    while time.perf_counter() - t0 < 3.0:
        oracle.transpose(x, threads=threads)
        reps += 1
    el = time.perf_counter() - t0
    return {"value": 2 * x.nbytes * reps / el / 1e9, "unit": "GB/s", "cores": threads, "kind": "oracle",
            "sample": f"{band} x {cols} row band of the {rows}x{cols} matrix, naive oracle transpose, "
                      f"{reps} reps in {el:.1f} s"}


def cpu_baseline_sweep():
    import oracle
    threads = oracle.max_threads()
    n, reps, t0 = 20000, 0, time.perf_counter()
    while time.perf_counter() - t0 < 3.0:
        oracle.sweep(32, ALL_PAT, SCH, 1, reps * n, n, threads=threads)
        reps += 1
    el = time.perf_counter() - t0
    return {"value": n * reps / el, "unit": "trials/s", "cores": threads, "kind": "oracle",
            "sample": f"{n * reps} trials of the w=32 sweep (5 patterns x RAW/RAS/RAP) in {el:.1f} s"}


def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)
    if args.gpus > 1 or args.workload == "dist":
        from paper_conf_icppw_nakanomi14_b200 import bench_dist
        return bench_dist.main(args)
    import torch

    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_icppw_nakanomi14_b200 as rap
    import workloads

    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    stream = torch.cuda.current_stream()
    peak, peak_src = load_peaks()

    if args.workload == "cfg4":
        rows = cols = 16384
        dt, dname, layouts = torch.float64, "u64", [args.layout]
    elif args.workload == "tile":
        rows = cols = 32
        dt, dname, layouts = torch.float32, "u32", [args.layout]
    else:
        rows = cols = 8192
        dt, dname, layouts = torch.float32, "u32", [args.layout]
    if args.workload == "layouts":
        layouts = ["raw", "pad", "xor", "ras", "rap"]
    do_t = args.workload != "sweep"
    do_s = args.workload in ("default", "sweep")
    eb = torch.empty((), dtype=dt).element_size()
    nbytes = 2 * rows * cols * eb

    x = workloads.random_bits(rows, cols, dt, seed=0, device=dev) if do_t else None
    y = torch.empty((cols, rows), dtype=dt, device=dev) if do_t else None
    hist = torch.zeros((5, 3, 33), dtype=torch.int64, device=dev)
    S = args.sweep_trials

    results = {}
    for lay in layouts:
        launches = 0
        ev = []
        trial0 = 0
        for k in range(args.warmup):
            if do_t:
                rap.transpose(x, layout=lay, seed=0, out=y)
            if do_s:
                rap.congestion_sweep(S, seed=1, first_trial=trial0, out=hist, algo=args.sweep_algo)
                trial0 += S
        torch.cuda.synchronize()
        hist.zero_()
        trial0 = 0
        with Clocks(0) as clk:
            start = torch.cuda.Event(enable_timing=True)
            end = torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            start.record(stream)
            for k in range(args.steps):
                e = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
                e[0].record(stream)
                if do_t:
                    rap.transpose(x, layout=lay, seed=0, out=y)
                    launches += 1
                e[1].record(stream)
                e[2].record(stream)
                if do_s:
                    rap.congestion_sweep(S, seed=1, first_trial=trial0, out=hist, algo=args.sweep_algo)
                    trial0 += S
                    launches += 1
                e[3].record(stream)
                ev.append(e)
            end.record(stream)
            torch.cuda.synchronize()
        total_ms = start.elapsed_time(end)
        t_ms = [e[0].elapsed_time(e[1]) for e in ev]
        s_ms = [e[2].elapsed_time(e[3]) for e in ev]
        results[lay] = dict(total_ms=total_ms, t_ms=t_ms, s_ms=s_ms, clocks=clk.result, launches=launches)

    lay = args.layout if args.workload != "layouts" else "rap"
    r = results[lay]
    line = {"metric": METRIC, "n_gpus": 1, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": r["total_ms"] / args.steps, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": dname, "data": "synthetic"}
    if do_t:
        avg_t = sum(r["t_ms"]) / len(r["t_ms"])
        gbs = nbytes / (avg_t * 1e-3) / 1e9
        line.update(value=gbs, unit="GB/s")
        line["config"] = {"workload": {"default": "cfg3 8192x8192 float32 RAP transpose + cfg2 w=32 sweep batch",
                                       "cfg4": "cfg4 16384x16384 float64 RAP transpose",
                                       "tile": "cfg1 32x32 float32 RAP tile",
                                       "layouts": "cfg3 8192x8192 float32 transpose, 5 smem layouts"}[args.workload],
                          "rows": rows, "cols": cols, "elem_bytes": eb, "layout": lay,
                          "l2": "inputs larger than L2 (no flush)" if nbytes // 2 > 126e6 else "L2-resident (latency case)",
                          "algorithmic_bytes_per_step": nbytes}
        kkey = f"transpose_b{eb * 8}_{lay}"
        line["roofline"] = {"bound": "hbm", "achieved": gbs, "peak": peak, "unit": "GB/s",
                            "frac": gbs / peak, "traffic": load_traffic(kkey),
                            "peak_source": peak_src, "frac_of_8TBs_nominal": gbs / 8000.0,
                            "kernel": kkey, "kernel_ms_median": statistics.median(r["t_ms"])}
        if args.workload == "layouts":
            line["layouts_gbs"] = {l: nbytes / (sum(v["t_ms"]) / len(v["t_ms"]) * 1e-3) / 1e9
                                   for l, v in results.items()}
    if do_s:
        s_avg = sum(r["s_ms"]) / len(r["s_ms"])
        tps = S / (s_avg * 1e-3)
        h = hist.cpu().numpy()
        import numpy as np
        c = np.arange(33)
        E = lambda a: float((a * c).sum() / a.sum())
        sweep = {"trials_per_s": tps, "trials_per_step": S, "w": 32,
                 "E_ras_stride": E(h[1, 1]), "E_rap_diagonal": E(h[2, 2]), "E_random": E(h[3, 2]),
                 "E_raw_malicious": E(h[4, 0]), "E_rap_stride": E(h[1, 2]),
                 "kernel_ms_median": statistics.median(r["s_ms"])}
        line["sweep"] = sweep
        if not do_t:
            line.update(value=tps, unit="trials/s",
                        config={"workload": "cfg2 w=32 congestion sweep", "trials_per_step": S})
            line["roofline"] = {"bound": "alu", "achieved": None, "peak": None, "unit": "warp-instr/s",
                                "frac": None, "traffic": None,
                                "note": "issue-bound; see profiles/ for smsp__issue_active"}
    line["clocks"] = r["clocks"]
    line["gpu_launches"] = r["launches"]

    # ---- e2e: the same step through the public API with host buffers (pinned)
    if not args.no_e2e and do_t:
        hx = x.cpu().pin_memory()
        hy = torch.empty((cols, rows), dtype=dt).pin_memory()
        hh = torch.empty_like(hist, device="cpu").pin_memory()
        dx = torch.empty_like(x)
        for k in range(2):
            dx.copy_(hx, non_blocking=True)
            rap.transpose(dx, layout=lay, seed=0, out=y)
            hy.copy_(y, non_blocking=True)
        torch.cuda.synchronize()
        K = max(3, min(args.steps, 20))
        st = torch.cuda.Event(enable_timing=True)
        en = torch.cuda.Event(enable_timing=True)
        st.record(stream)
        for k in range(K):
            dx.copy_(hx, non_blocking=True)
            rap.transpose(dx, layout=lay, seed=0, out=y)
            hy.copy_(y, non_blocking=True)
            if do_s:
                rap.congestion_sweep(S, seed=1, first_trial=k * S, out=hist)
                hh.copy_(hist, non_blocking=True)
        en.record(stream)
        torch.cuda.synchronize()
        ms = st.elapsed_time(en) / K
        line["e2e"] = {"value": nbytes / (ms * 1e-3) / 1e9, "unit": "GB/s",
                       "h2d_bytes_per_step": hx.numel() * eb,
                       "d2h_bytes_per_step": hy.numel() * eb + (hh.numel() * 8 if do_s else 0),
                       "ms_per_step": ms, "steps": K,
                       "note": "pinned host in -> H2D -> rap.transpose -> D2H (+ sweep batch, histogram D2H)"}
        bd = torch.int32 if eb == 4 else torch.int64
        assert torch.equal(hy.view(bd), y.cpu().view(bd)), "e2e result differs from the device result"
    if not args.no_cpu:
        if do_t:
            line["cpu_baseline"] = cpu_baseline_transpose(rows, cols, dt)
        else:
            line["cpu_baseline"] = cpu_baseline_sweep()
        if do_s and do_t:
            line["sweep"]["cpu_baseline"] = cpu_baseline_sweep()
    print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
