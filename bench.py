"""bench.py -- RAP hot path on B200: one JSON line per run (driver contract).

Default step (BASELINE configs; DESIGN.md §7 "Measurement"): one pass of the whole hot path --
  T0-T3  RAP transpose of the cfg4 matrix: 16384 x 16384 float64 (the paper's 64-bit doubles,
         P:L855-866), out-of-place, RAP = the w = 32 map on two 32-bit planes; input and output
         are 2 GiB each (> the 126 MB L2: no flush between steps);
  C1-C4  a slice of the cfg2 congestion sweep (w = 32, 5 patterns x RAW/RAS/RAP, seed 1): step k
         sweeps trials [k*S, (k+1)*S), S = 2^20 (~0.3 ms, so the transpose stays the step's
         dominant kernel); after the timed steps one timed sweep call covers the rest of
         [0, 10^9), so the run's histogram is the full cfg2 result and is compared with the
         oracle's stored 10^9-trial histogram (tests/golden/sweep_w32_1e9_seed1.txt, written from
         oracle/ only);
  (N > 1) the NCCL all-reduce of each step's sweep histogram.
`value` = the cfg4 transpose (GB/s, whole job): algorithmic bytes (read once + write once) of all
ranks / mean transpose device time per step (CUDA events on the launching stream, max over
ranks); `roofline` is that kernel's, on the same mean.  Sub-objects timed in the same run:
  `sweep`       the 10^9-trial cfg2 sweep (trials/s, pipe roofline, parity with the golden file);
  `cfg3_layouts` cfg3 8192^2 float32 under RAW / PAD / XOR / RAS / RAP (back-to-back launches);
  `cfg4_layouts` cfg4 under every 64-bit layout (two 32-bit planes; RAP64 8-byte slots; RAP-16);
  `trace`        the access-trace evaluator (4096 synthetic trace warps x 2048 trials x 5 schemes);
  `cfg1_tile`    cfg1's single 32 x 32 tile (latency, CUDA-graph replay);
  `cfg5_single_gpu` the 32768^2 float32 transpose on one GPU (N = 1);
each with its roofline and `cpu_baseline` (the oracle, all cores and one core, same sample
definition as the reference arm).

--workload picks another timed step: cfg3 (the round-1 default: cfg3 transpose + a sweep
batch), sweep (cfg2 only; value = trials/s), cfg4 (cfg4 alone with the 64-bit ablations), tile
(cfg1 32 x 32), layouts (cfg3 under the five layouts), dist / dist_fused (cfg5 32768^2 float32
row-block-sharded over the ranks: NCCL all-to-all / fused peer stores), trace (access traces).
--impl reference times the CPU oracle (the only reference this paper has: it publishes no
code) on a bounded sample of the same workload on the host cores; rank 0 only.

N > 1 (torchrun, one process per GPU): every rank transposes its own cfg4 matrix (replicas,
weak scaling) and sweeps its slice of each step's trial batch (the 10^9 trials are split over
the ranks; one all-reduce per step); `dist` shards one matrix (strong scaling).
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
NVLINK_GBS = 770.0   # measured peer copy per direction (B200_PROFILING.md); 900 nominal
SWEEP_TOTAL = 10 ** 9          # cfg2: trials swept by the default run (timed steps + the sweep sub-run)
STEP_SWEEP_TRIALS = 1 << 20    # default step's sweep slice: ~0.3 ms, so the cfg4 transpose stays the
                               # step's dominant kernel (its roofline is the line's `roofline`)
SWEEP_SEED = 1
CFG3_LAYOUTS = ["raw", "pad", "xor", "ras", "rap"]
CFG4_LAYOUTS = ["raw", "pad", "xor", "ras", "rap", "rap64", "rap16"]
# the cfg4 headline's 64-bit RAP encoding: the paper's w = 32 map with one double per 8-byte slot
# (DESIGN reading xv; 2.00 wavefronts per 256-byte request, the minimum) -- the two-plane and
# RAP-16 encodings are timed beside it in `cfg4_layouts`
HEADLINE64 = "rap64"
ORACLE_BAND_BYTES = 32 << 20   # the oracle's transpose sample: one row band of this many bytes,
ORACLE_PASSES = 8              # transposed this many times per step: one ~2 ms pass per step left the
#   two arms 20-25 % apart on the same box (thread start-up noise); one 256 MiB band per step measured
#   the oracle 5x slower (6 vs 32-40 GB/s: its naive column writes then thrash the caches)
E2E_WS = 64 << 20              # device workspace of the cfg4 host-to-host transpose: 4 band buffers of
                               # 128 rows (profiles/r02_e2e_bands.txt: the fastest band plan for cfg4)


# The JSON line goes to the process's original stdout; everything else that native code prints
# on fd 1 (NCCL's "NCCL version" banner, NCCL_DEBUG=INFO lines) is sent to stderr, so rank 0's
# stdout carries exactly one line.
_JSON_OUT = None


def emit(line: dict):
    global _JSON_OUT
    out = _JSON_OUT if _JSON_OUT is not None else sys.stdout
    out.write(json.dumps(line) + "\n")
    out.flush()


def route_native_stdout_to_stderr():
    global _JSON_OUT
    if _JSON_OUT is None:
        sys.stdout.flush()
        _JSON_OUT = os.fdopen(os.dup(1), "w")
        os.dup2(2, 1)


def parse(argv=None):
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=20)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--impl", default="mine", choices=["mine", "reference"])
    p.add_argument("--workload", default="default",
                   choices=["default", "cfg3", "sweep", "trace", "cfg4", "tile", "layouts", "dist", "dist_fused"])
    # --workload cfg3: one batch of 32 trials for every resident warp of the sweep kernel on a
    # B200 (148 SMs x 8 CTAs x 4 warps) per step.  `--workload sweep` (cfg2) defaults to 64
    # batches per warp (9.7 M trials, ~3 ms per step): the steady rate.  The default workload
    # sweeps ceil(10^9 / steps) trials per step instead.
    p.add_argument("--sweep-trials", type=int, default=None)
    # --workload trace: each of the 4096 trace warps evaluated under this many trials per step
    # (2048: a 0.6 ms launch, past the launch ramp; 256 trials run at ~80 % of that rate)
    p.add_argument("--trace-trials", type=int, default=2048)
    p.add_argument("--sweep-algo", default="default", choices=["default", "match"])
    p.add_argument("--layout", default="rap")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-cpu", action="store_true")
    a = p.parse_args(argv)
    if a.sweep_trials is None:
        if a.workload == "default":
            a.sweep_trials = STEP_SWEEP_TRIALS
        else:
            a.sweep_trials = 148 * 8 * 4 * 32 * (64 if a.workload == "sweep" else 1)
    return a


def dist_env():
    return (int(os.environ.get("WORLD_SIZE", "1")), int(os.environ.get("RANK", "0")),
            int(os.environ.get("LOCAL_RANK", "0")))


def load_peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(path):
        d = json.load(open(path))
        return float(d["hbm_gbs"]), "measured: MEASURED_PEAKS.json hbm_gbs (torch copy_, 2 GiB)"
    return 6650.0, "fallback: B200_PROFILING.md 6.65 TB/s"


def load_profile(kernel_key: str):
    """Per-launch DRAM bytes and smem wavefronts/request from the committed ncu summary."""
    path = os.path.join(ROOT, "profiles", "ncu_summary.json")
    if not os.path.exists(path):
        return None
    return json.load(open(path)).get("kernels", {}).get(kernel_key)


def host_cpu() -> dict:
    """The host the oracle runs on: model name, logical CPUs, CPUs this process may use."""
    model = None
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                model = ln.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    try:
        usable = len(os.sched_getaffinity(0))
    except AttributeError:
        usable = os.cpu_count()
    return {"cpu_model": model, "nproc": usable, "logical_cpus": os.cpu_count()}


class Clocks:
    """nvidia-smi sampler running during the timed region (start before, stop after)."""

    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")
    NAMES = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]

    def __init__(self, index: int):
        self.index, self.proc, self.result = index, None, None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "20"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            time.sleep(0.1)    # nvidia-smi start-up; samples begin during the soak
        except OSError:
            self.proc = None
        return self

    def __exit__(self, *a):
        if self.proc is None:
            self.result = {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
            return
        self.proc.terminate()
        out, _ = self.proc.communicate(timeout=10)
        sm, mx, reasons = [], [], set()
        for ln in out.strip().splitlines():
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 7:
                continue
            try:
                sm.append(float(f[0]))
                mx.append(float(f[1]))
            except ValueError:
                continue
            for n, v in zip(self.NAMES, f[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        self.result = {"sm_mhz": statistics.median(sm) if sm else None,
                       "sm_max_mhz": max(mx) if mx else None, "reasons": sorted(reasons),
                       "samples": len(sm), "window": "timed steps + 0.3 s of identical untimed steps each side"}


def clocks_bad(c: dict) -> bool:
    """A timed region that saw thermal / hardware slowdown, or SM clocks well below max with no
    reason given (a leftover clock lock), is measured once more."""
    bad = bool(set(c.get("reasons") or []) & {"hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown"})
    return bad or bool(c.get("sm_mhz") and c.get("sm_max_mhz") and not c.get("reasons")
                       and c["sm_mhz"] < 0.85 * c["sm_max_mhz"])


# ---------------------------------------------------------------------------- workload config
DESC = {"default": "cfg4 16384x16384 float64 RAP transpose (w=32 map, one double per 8-byte slot) + cfg2 w=32 "
                   "sweep slice per step (2^20 trials; the rest of 10^9 in one timed call); sub-objects: cfg2 "
                   "sweep, cfg3 8192x8192 float32 under raw/pad/xor/ras/rap, cfg4 under every 64-bit layout, "
                   "cfg1 tile, cfg5 on one GPU",
        "cfg3": "cfg3 8192x8192 float32 RAP transpose + cfg2 w=32 sweep batch",
        "cfg4": "cfg4 16384x16384 float64 RAP transpose (w=32 map, one double per 8-byte slot)",
        "tile": "cfg1 32x32 float32 RAP tile (latency case)",
        "layouts": "cfg3 8192x8192 float32 transpose under 5 smem layouts",
        "dist": "cfg5 32768x32768 float32 row-block-sharded transpose over {world} GPU(s), NCCL all-to-all",
        "dist_fused": "cfg5 32768x32768 float32 row-block-sharded transpose over {world} GPU(s), "
                      "fused: tiles stored straight into peer shards (symmetric memory)",
        "sweep": "cfg2 w=32 congestion sweep, 5 patterns x RAW/RAS/RAP",
        "trace": "congestion of 4096 synthetic warp traces (row / column / diagonal / "
                 "anti-diagonal / permutation / random) under RAW, RAS, RAP, PAD, XOR"}


def transpose_shape(wl: str, world: int):
    """(rows per rank, cols, elem_bytes) of the workload's timed transpose."""
    if wl in ("default", "cfg4"):
        return 16384, 16384, 8
    if wl == "tile":
        return 32, 32, 4
    if wl in ("dist", "dist_fused"):
        return 32768 // world, 32768, 4
    return 8192, 8192, 4


def arm_config(args, world: int) -> dict:
    """The `config` object of the JSON line for args.workload -- one definition for both arms."""
    wl = args.workload
    if wl == "sweep":
        return {"workload": DESC[wl], "trials_per_step": args.sweep_trials * world,
                "parallelism": f"trial ranges x{world} + NCCL all-reduce" if world > 1 else "single GPU"}
    if wl == "trace":
        return {"workload": DESC[wl], "trials_per_step": args.trace_trials, "warps": 4096, "schemes": 5}
    rows_rank, n, eb = transpose_shape(wl, world)
    lay = (HEADLINE64 if wl == "default" or (wl == "cfg4" and args.layout == "rap")
           else "rap" if wl == "layouts" else args.layout)
    nbytes = 2 * rows_rank * n * eb
    cfg = {"workload": DESC[wl].format(world=world), "rows": n, "cols": n, "elem_bytes": eb, "layout": lay,
           "parallelism": (f"row blocks + NCCL all-to-all, {world} ranks" if wl == "dist"
                           else f"row blocks + NVLink peer stores, {world} ranks" if wl == "dist_fused"
                           else f"replicas x{world}" if world > 1 else "single GPU"),
           "l2": ("inputs larger than L2 (no flush)" if nbytes // 2 > 126e6
                  else "input fits in L2 (no flush; latency case)"),
           "algorithmic_bytes_per_step_per_rank": nbytes}
    if wl == "cfg3":
        cfg["sweep_trials_per_step"] = args.sweep_trials * world
    if wl == "default":
        cfg["sweep_trials_per_step"] = args.sweep_trials
        cfg["sweep_trials_total"] = SWEEP_TOTAL
        cfg["sweep_seed"] = SWEEP_SEED
    return cfg


# ---------------------------------------------------------------------------- oracle timing
def oracle_band(rows: int, cols: int, eb: int) -> int:
    """Rows of the oracle's transpose sample: one band of ORACLE_BAND_BYTES (both arms)."""
    return max(1, min(rows, ORACLE_BAND_BYTES // (cols * eb)))


def oracle_transpose_sample(rows: int, cols: int, dt):
    import workloads
    band = oracle_band(rows, cols, workloads_eb(dt))
    return workloads.as_bits_numpy(workloads.random_bits(band, cols, dt, seed=0)), band


def workloads_eb(dt) -> int:
    import torch
    return torch.empty((), dtype=dt).element_size()


def rate_for(fn, work: float, seconds: float):
    """Calls fn() for `seconds` (after one untimed call); returns (work per second, calls, elapsed)."""
    fn()
    reps, t0 = 0, time.perf_counter()
    while True:
        fn()
        reps += 1
        el = time.perf_counter() - t0
        if el >= seconds:
            return work * reps / el, reps, el


def cpu_baseline_transpose(rows, cols, dt, seconds: float = 3.0):
    """The oracle's naive transpose on one row band of the matrix: all cores (value) and one core."""
    import numpy as np

    import oracle
    threads = oracle.max_threads()
    x, band = oracle_transpose_sample(rows, cols, dt)
    out = np.empty((x.shape[1], x.shape[0]), dtype=x.dtype)
    gb = 2 * x.nbytes / 1e9
    v_all, n_all, t_all = rate_for(lambda: oracle.transpose(x, threads=threads, out=out), gb, seconds)
    v_one, n_one, t_one = rate_for(lambda: oracle.transpose(x, threads=1, out=out), gb, seconds)
    return dict({"value": v_all, "unit": "GB/s", "cores": threads, "kind": "oracle",
                 "sample": f"{band} x {cols} row band ({x.nbytes >> 20} MiB) of the {rows}x{cols} "
                           f"{str(dt)[6:]} matrix, naive oracle transpose into a reused output array; "
                           f"{n_all} calls in {t_all:.1f} s on {threads} threads, {n_one} in {t_one:.1f} s on 1",
                 "value_single_thread": v_one}, **host_cpu())


def cpu_baseline_tile(seconds: float = 1.0):
    """cfg1: the oracle transposing one 32 x 32 float32 tile (per-call time, one thread)."""
    import oracle
    import torch
    import workloads
    x = workloads.as_bits_numpy(workloads.random_bits(32, 32, torch.float32, seed=0))
    v, n, el = rate_for(lambda: oracle.transpose(x, threads=1), 1.0, seconds)
    return {"us_per_tile": 1e6 / v, "cores": 1, "kind": "oracle",
            "sample": f"32x32 float32 tile, {n} oracle calls in {el:.1f} s (includes the ctypes call)"}


def cpu_baseline_sweep(seconds: float = 3.0):
    import oracle
    threads = oracle.max_threads()
    n = 20000
    k = [0]

    def run(th):
        oracle.sweep(32, ALL_PAT, SCH, SWEEP_SEED, k[0] * n, n, threads=th)
        k[0] += 1
    v_all, n_all, t_all = rate_for(lambda: run(threads), n, seconds)
    v_one, n_one, t_one = rate_for(lambda: run(1), n, seconds)
    return dict({"value": v_all, "unit": "trials/s", "cores": threads, "kind": "oracle",
                 "sample": f"w=32 sweep (5 patterns x RAW/RAS/RAP), {n}-trial chunks: {n_all} in {t_all:.1f} s "
                           f"on {threads} threads, {n_one} in {t_one:.1f} s on 1",
                 "value_single_thread": v_one}, **host_cpu())


# ---------------------------------------------------------------------------- reference arm
def run_reference(args):
    """The CPU oracle, as it stands, on the host cores, on a bounded sample of the workload."""
    world, rank, _ = dist_env()
    if world > 1 and rank != 0:
        return
    emit(oracle_arm(args, world))


def oracle_arm(args, world: int, threads: int | None = None, workload: str | None = None) -> dict:
    """The reference arm's measurement (K steps of the workload's oracle sample after W warm-ups),
    as the JSON line `--impl reference` prints.  Our arm's `cpu_baseline` objects call the same
    function (same sample, same step structure), so the two agree up to box noise."""
    import numpy as np
    import torch

    import oracle
    threads = oracle.max_threads() if threads is None else threads
    wl = args.workload if workload is None else workload
    cfg = arm_config(args if workload is None else argparse.Namespace(**dict(vars(args), workload=wl)), world)
    n_sw = 20000                           # oracle sweep sample: trials per step

    def sweep_sample(k):
        oracle.sweep(32, ALL_PAT, SCH, SWEEP_SEED, k * n_sw, n_sw, threads=threads)

    sweep_s = 0.0
    if wl == "sweep":
        unit, what = "trials/s", f"{n_sw} trials of the w=32 sweep (5 patterns x RAW/RAS/RAP) per step"
        work = n_sw

        def fn(k):
            t = time.perf_counter()
            sweep_sample(k)
            t_steps.append(time.perf_counter() - t)
    elif wl == "trace":
        fn, work, what = oracle_trace_sample()
        unit = "warp-evaluations/s"
    else:
        rows_rank, cols, eb = transpose_shape(wl, 1)
        dt = torch.float64 if eb == 8 else torch.float32
        x, band = oracle_transpose_sample(rows_rank, cols, dt)
        out = np.empty((x.shape[1], x.shape[0]), dtype=x.dtype)
        unit = "GB/s"
        what = (f"{ORACLE_PASSES} passes over a {band} x {cols} row band ({x.nbytes >> 20} MiB) of the "
                f"{rows_rank}x{cols} {str(dt)[6:]} matrix per step, naive oracle transpose on {threads} threads "
                f"into a reused output array")
        if wl in ("default", "cfg3"):
            what += f"; plus {n_sw} oracle sweep trials per step, timed apart (`sweep`)"
        work = 2 * x.nbytes * ORACLE_PASSES / 1e9

        def fn(k):
            nonlocal sweep_s
            t = time.perf_counter()
            for _ in range(ORACLE_PASSES):
                oracle.transpose(x, threads=threads, out=out)
            t_steps.append(time.perf_counter() - t)
            if wl in ("default", "cfg3"):        # the step's second half, timed apart like our arm's
                t = time.perf_counter()
                sweep_sample(k)
                sweep_s += time.perf_counter() - t
                s_steps.append(time.perf_counter() - t)
    t_steps, s_steps = [], []
    for k in range(args.warmup):
        fn(k)
    sweep_s = 0.0
    t_steps, s_steps = [], []
    t0 = time.perf_counter()
    for k in range(args.steps):
        fn(args.warmup + k)
    el = time.perf_counter() - t0
    # the median step: the host cores are shared, and one step that loses its cores to another
    # process should not set the baseline (our arm's cpu_baseline uses the same function)
    value = (work / statistics.median(t_steps) if t_steps
             else work * args.steps / (el - sweep_s))
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": unit, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": el / args.steps * 1e3,
            "higher_is_better": True, "scaling": "strong" if wl in ("dist", "dist_fused") else "weak",
            "vs_baseline": None, "dtype": "u64" if wl in ("cfg4", "default") else "u32", "data": "synthetic",
            "config": cfg,
            "cpu_baseline": dict({"value": value, "unit": unit, "cores": 1 if wl == "trace" else threads,
                                  "kind": "oracle", "sample": what}, **host_cpu()),
            "e2e": {"value": value, "unit": unit, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    if wl in ("default", "cfg3"):
        line["sweep"] = {"trials_per_s": n_sw / statistics.median(s_steps), "trials_per_step": n_sw}
    line["cpu_baseline"]["statistic"] = "median step" if t_steps or s_steps else "total time"
    return line


def oracle_trace_sample():
    """(fn(k), evaluations per call, description): the oracle's direct DMM congestion (O8) per
    (trace warp, trial, scheme), as the parity test computes it -- 64 of the 4096 trace warps x
    4 trials x 5 schemes per call."""
    import oracle
    import workloads
    cells = workloads.trace_cells(4096, 32, seed=0).numpy()[:64]
    sch5 = ["raw", "ras", "rap", "pad", "xor"]

    def fn(k):
        for n in range(4 * k, 4 * k + 4):
            P, r = oracle.perm(1, n, 32), oracle.ras_shifts(1, n, 32)
            for cw in cells:
                for s in sch5:
                    oracle.congestion(32, cw // 32, cw % 32, oracle.SCHEMES[s], {"ras": r, "rap": P}.get(s))
    return fn, 64 * 4 * 5, "64 of the 4096 trace warps x 4 trials x 5 schemes per call, oracle congestion (O8) one by one"


def cpu_baseline_trace():
    fn, work, what = oracle_trace_sample()
    k = [0]

    def call():
        fn(k[0])
        k[0] += 1
    v, reps, el = rate_for(call, work, 3.0)
    return dict({"value": v, "unit": "warp-evaluations/s", "cores": 1, "kind": "oracle",
                 "sample": f"{what}; {reps} calls in {el:.1f} s (single thread: one ctypes call per evaluation)"},
                **host_cpu())


def _capture_pipes(prof: dict):
    """(pipe-active fractions, capture duration s) of the committed ncu capture (exported raw page)."""
    src = (prof or {}).get("source", "")
    path = os.path.join(ROOT, src.split()[0].replace(".ncu-rep[.gz]", ".raw.csv")) if src else ""
    if not path.endswith(".raw.csv") or not os.path.exists(path):
        return None, None
    import csv
    rows = list(csv.reader(open(path)))
    h, u, v = rows[0], rows[1], rows[2]
    fr = {}
    for pipe in ("alu", "adu", "fma", "lsu", "xu"):
        key = f"sm__inst_executed_pipe_{pipe}.avg.pct_of_peak_sustained_active"
        if key in h:
            fr[pipe] = float(v[h.index(key)].replace(",", "")) / 100
    key = "smsp__issue_active.avg.pct_of_peak_sustained_active"
    if key in h:
        fr["issue"] = float(v[h.index(key)].replace(",", "")) / 100
    k = "gpu__time_duration.sum"
    dur = None
    if k in h:
        scale = {"ns": 1e-9, "nsecond": 1e-9, "us": 1e-6, "usecond": 1e-6, "ms": 1e-3, "msecond": 1e-3, "s": 1.0}
        dur = float(v[h.index(k)].replace(",", "")) * scale.get(u[h.index(k)], 1.0)
    return fr, dur


def pipe_roofline(rate: float, unit: str, prof_key: str, what: str) -> dict:
    """Roofline of an integer kernel against its busiest pipe.  The committed ncu capture gives,
    per pipe (ALU: LOP3 / SHF / IADD3 / SEL ...; ADU: CREDUX / VOTE / MATCH; FMA: IMAD; LSU:
    shared memory, shuffles; the issue slots, 1 warp-instruction / clk / SMSP), the fraction of its
    peak the kernel used at the
    capture's rate; peak = the rate at which the busiest pipe would be 100 % busy with the same
    instruction mix (capture rate / that fraction); achieved = the live rate; frac = achieved / peak.
    The ALU-pipe view of round 1 (148 SMs x 4 SMSPs x 0.5 warp-instr/clk) is in `pipes`."""
    prof = load_profile(prof_key) or {}
    fr, dur = _capture_pipes(prof)
    units = (prof.get("units_per_launch") or {})
    n = next(iter(units.values()), None)
    if not fr or not dur or not n:
        return {"bound": "alu", "achieved": rate, "peak": None, "unit": unit, "frac": None, "traffic": None,
                "note": "no committed ncu capture"}
    cap_rate = n / dur
    pipe = max(fr, key=lambda p: fr[p])                 # the issue slots count as a pipe too
    peak = cap_rate / fr[pipe]
    return {"bound": pipe, "achieved": rate, "peak": peak, "unit": unit, "frac": rate / peak, "traffic": None,
            "pipes_active_at_capture": fr, "capture_rate": cap_rate,
            "peak_source": f"ncu capture {prof.get('source', '').split()[0]}: {what} rate at which the {pipe.upper()} "
                           f"pipe (the busiest) is 100% busy = capture rate / its active fraction",
            "alu_warp_instructions_per_unit": prof.get("alu_warp_instructions_per_trial",
                                                        prof.get("alu_warp_instructions_per_evaluation")),
            "warp_instructions_per_unit": prof.get("warp_instructions_per_trial",
                                                    prof.get("warp_instructions_per_evaluation"))}


def sweep_roofline(tps: float, clocks: dict):
    """The sweep against its busiest pipe (pipe_roofline; the ADU since the bank counters)."""
    return pipe_roofline(tps, "trials/s", "sweep_w32", "trial")


def trace_roofline(eps: float, clocks: dict):
    """The trace evaluator against its busiest pipe (pipe_roofline)."""
    r = pipe_roofline(eps, "warp-evaluations/s", "trace_w32", "warp-evaluation")
    r["traffic"] = (load_profile("trace_w32") or {}).get("dram_bytes_per_launch")
    return r


def hbm_roofline(nbytes: int, ms: float, peak: float, peak_src: str, kkey: str) -> dict:
    """HBM roofline of one transpose launch: algorithmic bytes / mean launch time."""
    prof = load_profile(kkey) or {}
    ach = nbytes / (ms * 1e-3) / 1e9
    return {"bound": "hbm", "achieved": ach, "peak": peak, "unit": "GB/s", "frac": ach / peak,
            "traffic": prof.get("dram_bytes_per_launch_steady", prof.get("dram_bytes_per_launch")),
            "peak_source": peak_src, "frac_of_8TBs_nominal": ach / 8000.0, "kernel": kkey,
            "kernel_name": prof.get("kernel_name"), "kernel_ms_mean": ms, "algorithmic_bytes_per_launch": nbytes,
            "smem_wavefronts_per_request": prof.get("smem_wavefronts_per_request"),
            "profile": prof.get("source")}


def reduce_over_ranks(x: float, world: int, dev, op: str) -> float:
    if world == 1:
        return x
    import torch
    import torch.distributed as dist
    t = torch.tensor([x], dtype=torch.float64, device=dev if dist.get_backend() == "nccl" else "cpu")
    dist.all_reduce(t, op=dist.ReduceOp.MAX if op == "max" else dist.ReduceOp.SUM)
    return float(t.item())


def golden_sweep_1e9(seed: int):
    """The oracle's stored 10^9-trial cfg2 histogram [5][3][33] (tests/golden, written by
    tools/oracle_golden_1e9.py from oracle/ only), or None."""
    import numpy as np
    path = os.path.join(ROOT, "tests", "golden", f"sweep_w32_1e9_seed{seed}.txt")
    if not os.path.exists(path):
        return None
    rows = [ln.split() for ln in open(path) if ln.strip() and not ln.startswith("#")]
    h = np.array([[int(v) for v in r[2:]] for r in rows], dtype=np.uint64)
    return h.reshape(5, 3, 33)


# ---------------------------------------------------------------------------- our arm: default
def init_dist(world: int, dev, force: bool = False):
    """One process per GPU over NCCL; RAP_BENCH_BACKEND=gloo lets several ranks share one GPU to
    exercise the multi-rank code paths on a single-GPU box (NCCL refuses duplicate devices)."""
    import torch.distributed as dist
    if world > 1 or force:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("MASTER_PORT", "29571")
        os.environ.setdefault("RANK", "0")
        os.environ.setdefault("WORLD_SIZE", "1")
        backend = os.environ.get("RAP_BENCH_BACKEND", "nccl")
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)


def all_reduce_hist(h, world: int):
    """Sum a histogram over the ranks (NCCL on device; gloo via host memory)."""
    if world == 1:
        return
    import torch.distributed as dist
    if dist.get_backend() == "nccl":
        dist.all_reduce(h)
    else:
        hc = h.cpu()
        dist.all_reduce(hc)
        h.copy_(hc)


def soak_for(seconds: float, body, world: int, dev):
    """Runs body(k) (k = 0, 1, ...) for about `seconds` of wall time with the device synchronised
    after each call.  At N > 1 every rank runs the SAME number of calls -- the count comes from the
    first call's duration, max over ranks -- because a body may hold collectives (the sweep's
    all-reduce, the sharded transpose's all-to-all): a loop on each rank's own clock could leave
    the ranks a collective apart (a gloo size mismatch, an NCCL hang)."""
    import math
    import torch
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    body(0)
    torch.cuda.synchronize()
    dt = max(time.perf_counter() - t0, 1e-6)
    n = max(1, int(math.ceil(seconds / dt)))
    n = int(reduce_over_ranks(float(n), world, dev, "max"))
    for k in range(1, n):
        body(k)
        torch.cuda.synchronize()


def timed_back_to_back(fn, warmup: int, steps: int, stream, world: int, dev, barrier):
    """Mean device time of one fn() over `steps` back-to-back launches between one event pair
    (max over ranks), with the clocks sampled over them."""
    import torch
    for _ in range(warmup):
        fn()
    torch.cuda.synchronize()
    barrier()
    with Clocks(dev.index) as clk:
        soak_for(0.2, lambda k: fn(), world, dev)  # soak, so every clock sample is under load
        st, en = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        st.record(stream)
        for _ in range(steps):
            fn()
        en.record(stream)
        torch.cuda.synchronize()
    return reduce_over_ranks(st.elapsed_time(en), world, dev, "max") / steps, clk.result


def run_default(args):
    import numpy as np
    import torch
    import torch.distributed as dist

    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_icppw_nakanomi14_b200 as rap
    import workloads

    world, rank, local = dist_env()
    dev = torch.device("cuda", local % torch.cuda.device_count())
    torch.cuda.set_device(dev)
    init_dist(world, dev)
    stream = torch.cuda.current_stream()
    peak, peak_src = load_peaks()
    barrier = (lambda: dist.barrier()) if world > 1 else (lambda: None)
    rmax = lambda v: reduce_over_ranks(v, world, dev, "max")
    K, W = args.steps, args.warmup

    # ---------------- cfg4 headline + cfg2 sweep slices
    rows = cols = 16384
    dt = torch.float64
    nbytes = 2 * rows * cols * 8                     # per rank per step
    x = workloads.random_bits(rows, cols, dt, seed=rank, device=dev)
    y = torch.empty((cols, rows), dtype=dt, device=dev)
    S = args.sweep_trials                            # trials per step (all ranks together)
    total = min(SWEEP_TOTAL, S * K)                  # swept by the timed steps; the rest of the 10^9
                                                     # in the timed sweep sub-run below
    hist = torch.zeros((5, 3, 33), dtype=torch.int64, device=dev)
    hstep = torch.zeros_like(hist)
    scratch = torch.zeros_like(hist)

    def sweep_slice(first: int, n: int, out):
        """This rank's part of trials [first, first + n) into `out` (+ the all-reduce at N > 1)."""
        lo = first + n * rank // world
        hi = first + n * (rank + 1) // world
        if world == 1:
            rap.congestion_sweep(hi - lo, seed=SWEEP_SEED, first_trial=lo, out=out)
            return 1
        hstep.zero_()
        rap.congestion_sweep(hi - lo, seed=SWEEP_SEED, first_trial=lo, out=hstep)
        all_reduce_hist(hstep, world)                # the sweep's one exchange
        out.add_(hstep)
        return 1

    def soak(seconds, k0):
        def body(k):
            rap.transpose(x, layout=HEADLINE64, seed=0, out=y)
            sweep_slice((1 << 40) + (k0 + k) * S, S, scratch)    # far trial range, scratch histogram
        soak_for(seconds, body, world, dev)                       # (the same count on every rank)

    for k in range(W):
        rap.transpose(x, layout=HEADLINE64, seed=0, out=y)
        sweep_slice((1 << 41) + k * S, S, scratch)
    torch.cuda.synchronize()
    first_clocks = None
    for attempt in range(2):
        hist.zero_()
        launches, ev = 0, []
        barrier()
        torch.cuda.synchronize()
        with Clocks(dev.index) as clk:
            soak(0.3, 0)
            barrier()
            start = torch.cuda.Event(enable_timing=True)
            end = torch.cuda.Event(enable_timing=True)
            start.record(stream)
            for k in range(K):
                e = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
                e[0].record(stream)
                rap.transpose(x, layout=HEADLINE64, seed=0, out=y)          # T0-T3
                launches += 1
                e[1].record(stream)
                e[2].record(stream)
                n = min(S, total - k * S)
                if n > 0:
                    launches += sweep_slice(k * S, n, hist)             # C1-C4
                e[3].record(stream)
                ev.append(e)
            end.record(stream)
            torch.cuda.synchronize()
            barrier()
            soak(0.3, 1000)
        t_ms = [e[0].elapsed_time(e[1]) for e in ev]
        s_ms = [e[2].elapsed_time(e[3]) for e in ev]
        c = clk.result
        if attempt == 0 and rmax(1.0 if clocks_bad(c) else 0.0) > 0:
            first_clocks = c
            continue
        if first_clocks is not None:
            c = dict(c, remeasured=True, first_attempt=first_clocks)
        break
    total_ms, t_sum, s_sum = rmax(start.elapsed_time(end)), rmax(sum(t_ms)), rmax(sum(s_ms))
    kern_ms = t_sum / K                                           # mean transpose launch
    line = {"metric": METRIC, "n_gpus": world, "steps": K, "warmup": W, "ms_per_step": total_ms / K,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u64",
            "data": "synthetic (seeded random bit patterns; sweep trials are counters)",
            "value": nbytes * world / (kern_ms * 1e-3) / 1e9, "unit": "GB/s",
            "config": arm_config(args, world)}
    line["roofline"] = hbm_roofline(nbytes, kern_ms, peak, peak_src, f"transpose_b64_{HEADLINE64}")
    line["roofline"]["kernel_ms_median"] = rmax(statistics.median(t_ms))

    line["kernel_time_share"] = {"transpose": t_sum / (t_sum + s_sum), "sweep": s_sum / (t_sum + s_sum)}
    line["clocks"] = c
    line["gpu_launches"] = int(reduce_over_ranks(launches, world, dev, "sum"))

    # ---------------- sweep sub-object: the rest of cfg2's 10^9 trials (the steps swept
    # [0, K*S)), timed as one sweep of [K*S, 10^9) into the same histogram, then the whole
    # 10^9-trial histogram against the oracle's stored one
    rest = SWEEP_TOTAL - total
    barrier()
    torch.cuda.synchronize()
    with Clocks(dev.index) as sclk:
        st_, en_ = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        st_.record(stream)
        if rest > 0:
            sweep_slice(total, rest, hist)
        en_.record(stream)
        torch.cuda.synchronize()
    rest_ms = rmax(st_.elapsed_time(en_))
    h = hist.cpu().numpy().astype(np.uint64)
    cc = np.arange(33)
    E = lambda a: float((a * cc).sum() / a.sum())
    assert (h.sum(-1) == SWEEP_TOTAL).all(), "histogram does not hold every trial once"
    tps = rest / (rest_ms * 1e-3) if rest > 0 else total / (s_sum * 1e-3)
    gold = golden_sweep_1e9(SWEEP_SEED)
    line["sweep"] = {"trials_per_s": tps, "unit": "trials/s", "trials": SWEEP_TOTAL, "w": 32, "seed": SWEEP_SEED,
                     "timing": f"trials [0, {total}) in the {K} timed steps ({S} per step), [{total}, 10^9) in one "
                               "timed sweep call; trials_per_s is the latter's",
                     "trials_per_s_in_steps": total / (s_sum * 1e-3), "sub_run_ms": rest_ms,
                     "scaling": "strong (every call's trial range is split over the ranks)",
                     "E_ras_stride": E(h[1, 1]), "E_rap_diagonal": E(h[2, 2]), "E_random": E(h[3, 2]),
                     "E_raw_malicious": E(h[4, 0]), "E_rap_stride": E(h[1, 2]),
                     "bit_identical_to_oracle_1e9": (bool(np.array_equal(h, gold)) if gold is not None else None),
                     "oracle_reference": "tests/golden/sweep_w32_1e9_seed1.txt (oracle/, 10^9 trials)",
                     "clocks": sclk.result, "roofline": sweep_roofline(tps / world, sclk.result)}
    if gold is not None:
        assert np.array_equal(h, gold), "10^9-trial histogram differs from the oracle's"

    # ---------------- cfg3 under the five layouts, cfg4 under every 64-bit layout
    subs = {}
    x3 = workloads.random_bits(8192, 8192, torch.float32, seed=rank, device=dev)
    y3 = torch.empty_like(x3)
    for name, xx, yy, lays in (("cfg3_layouts", x3, y3, CFG3_LAYOUTS), ("cfg4_layouts", x, y, CFG4_LAYOUTS)):
        eb = xx.element_size()
        nb = 2 * xx.numel() * eb
        res = {}
        for lay in lays:
            ms, ck = timed_back_to_back(lambda: rap.transpose(xx, layout=lay, seed=0, out=yy), W, K, stream,
                                        world, dev, barrier)
            r = hbm_roofline(nb, ms, peak, peak_src, f"transpose_b{eb * 8}_{lay}")
            res[lay] = {"value": nb * world / (ms * 1e-3) / 1e9, "unit": "GB/s", "frac": r["frac"],
                        "kernel_ms_mean": ms, "smem_wavefronts_per_request": r["smem_wavefronts_per_request"],
                        "traffic": r["traffic"], "kernel_name": r["kernel_name"], "sm_mhz": ck.get("sm_mhz"),
                        "reasons": ck.get("reasons")}
        hl = "rap" if eb == 4 else HEADLINE64          # the layout whose roofline heads the sub-object
        sub = {"workload": ("cfg3 8192x8192 float32" if eb == 4 else "cfg4 16384x16384 float64"),
               "timing": f"{K} back-to-back launches per layout between one event pair (after {W} warm-ups)",
               "algorithmic_bytes_per_launch": nb, "layouts": res,
               "roofline": hbm_roofline(nb, res[hl]["kernel_ms_mean"], peak, peak_src, f"transpose_b{eb * 8}_{hl}")}
        subs[name] = sub
    del x3, y3
    line.update(subs)

    # ---------------- access traces (north star: "synthetic matrices and access traces"): 4096
    # trace warps of the paper's pattern families, each evaluated under 2048 trials and 5 schemes
    # per launch; K back-to-back launches over disjoint trial ranges
    cells = workloads.trace_cells(4096, 32, seed=rank, device=dev)
    th = torch.zeros((5, 33), dtype=torch.int64, device=dev)
    sch5 = ("raw", "ras", "rap", "pad", "xor")
    tk = [0]

    def trace_launch():
        rap.congestion_trace(cells, 2048, seed=1, schemes=sch5, first_trial=tk[0] * 2048, out=th)
        tk[0] += 1
    ms_t, ck_t = timed_back_to_back(trace_launch, W, K, stream, world, dev, barrier)
    evs = 4096 * 2048 * 5 / (ms_t * 1e-3)
    thc = th.cpu().numpy()
    cc33 = np.arange(33)
    line["trace"] = {"warp_evaluations_per_s": evs * world, "unit": "warp-evaluations/s",
                     "ras_rap_evaluations_per_s": evs * world * 2 / 5, "kernel_ms_mean": ms_t,
                     "per_launch": "4096 trace warps x 2048 trials x 5 schemes",
                     "E_by_scheme": {n: float((thc[i] * cc33).sum() / thc[i].sum()) for i, n in enumerate(sch5)},
                     "roofline": trace_roofline(evs, ck_t)}
    del cells, th

    # ---------------- cfg1: one 32 x 32 float32 tile (latency case: CUDA-graph replay of 256 launches)
    x1 = workloads.random_bits(32, 32, torch.float32, seed=rank, device=dev)
    y1 = torch.empty_like(x1)
    g = torch.cuda.CUDAGraph()
    cs = torch.cuda.Stream()
    cs.wait_stream(stream)
    with torch.cuda.stream(cs):
        rap.transpose(x1, layout="rap", seed=0, out=y1)
        torch.cuda.synchronize()
        with torch.cuda.graph(g, stream=cs):
            for _ in range(256):
                rap.transpose(x1, layout="rap", seed=0, out=y1)
    g.replay()
    torch.cuda.synchronize()
    gs, ge = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    gs.record(stream)
    for _ in range(10):
        g.replay()
    ge.record(stream)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(200):
        rap.transpose(x1, layout="rap", seed=0, out=y1)
    torch.cuda.synchronize()
    line["cfg1_tile"] = {"us_per_transpose_cuda_graph": rmax(gs.elapsed_time(ge)) * 1e3 / 2560,
                         "us_per_call_python": (time.perf_counter() - t0) / 200 * 1e6,
                         "note": "latency case, no roofline: one single-warp CTA, P from the host call"}

    # ---------------- cfg5 on one GPU: the 32768^2 float32 transpose the sharded path splits
    if world == 1:
        del x, y
        x5 = workloads.random_bits(32768, 32768, torch.float32, seed=rank, device=dev)
        y5 = torch.empty_like(x5)
        nb5 = 2 * x5.numel() * 4
        ms5, ck5 = timed_back_to_back(lambda: rap.transpose(x5, layout="rap", seed=0, out=y5), W, K, stream,
                                      world, dev, barrier)
        r5 = hbm_roofline(nb5, ms5, peak, peak_src, "transpose_b32_rap")
        line["cfg5_single_gpu"] = {"value": nb5 / (ms5 * 1e-3) / 1e9, "unit": "GB/s", "frac": r5["frac"],
                                   "kernel_ms_mean": ms5, "algorithmic_bytes_per_launch": nb5,
                                   "note": "32768^2 float32 RAP transpose on one GPU, back to back (the sharded "
                                           "cfg5 runs with --workload dist / dist_fused under torchrun)"}
        del x5, y5
        x = workloads.random_bits(rows, cols, dt, seed=rank, device=dev)
        y = torch.empty((cols, rows), dtype=dt, device=dev)

    # ---------------- e2e through the public API with pinned host buffers
    if not args.no_e2e:
        KE = max(3, min(K, 10))
        hx = x.cpu().pin_memory()
        hy = torch.empty((cols, rows), dtype=dt).pin_memory()
        for _ in range(2):
            rap.transpose_host(hx, out=hy, layout=HEADLINE64, seed=0, device=dev, workspace_bytes=E2E_WS)
        barrier()
        st = torch.cuda.Event(enable_timing=True)
        en = torch.cuda.Event(enable_timing=True)
        st.record(stream)
        for _ in range(KE):
            rap.transpose_host(hx, out=hy, layout=HEADLINE64, seed=0, device=dev, workspace_bytes=E2E_WS)
        en.record(stream)
        torch.cuda.synchronize()
        ms = rmax(st.elapsed_time(en)) / KE
        rap.transpose(x, layout=HEADLINE64, seed=0, out=y)
        assert torch.equal(hy.view(torch.int64), y.cpu().view(torch.int64)), "e2e result differs from the device result"
        line["e2e"] = {"value": nbytes * world / (ms * 1e-3) / 1e9, "unit": "GB/s",
                       "h2d_bytes_per_step": hx.numel() * 8 * world, "d2h_bytes_per_step": hy.numel() * 8 * world,
                       "ms_per_step": ms, "steps": KE,
                       "note": "rap_transpose_host: pinned host cfg4 matrix in, pinned host transpose out; "
                               f"upload / RAP transpose / download of row bands ({E2E_WS >> 20} MiB workspace) "
                               "overlapped"}
        del hx, hy
    if rank == 0 and not args.no_cpu and world == 1:
        # the reference arm's own measurement (oracle_arm), all host cores, plus one core
        ref = oracle_arm(args, 1)
        one = oracle_arm(args, 1, threads=1)
        cb = dict(ref["cpu_baseline"], value_single_thread=one["value"],
                  sample=ref["cpu_baseline"]["sample"] + f"; {args.steps} steps after {args.warmup} warm-ups "
                         "(the --impl reference measurement); value_single_thread: the same on 1 thread")
        line["cpu_baseline"] = cb
        line["sweep"]["cpu_baseline"] = dict({"value": ref["sweep"]["trials_per_s"], "unit": "trials/s",
                                               "cores": cb["cores"], "kind": "oracle",
                                               "value_single_thread": one["sweep"]["trials_per_s"],
                                               "sample": f"{ref['sweep']['trials_per_step']} oracle trials of the "
                                                         "w=32 sweep per step (the --impl reference step)"},
                                              **host_cpu())
        c3 = oracle_arm(args, 1, workload="cfg3")
        line["cfg3_layouts"]["cpu_baseline"] = dict(c3["cpu_baseline"], value_single_thread=oracle_arm(
            args, 1, threads=1, workload="cfg3")["value"])
        line["cfg1_tile_cpu_baseline"] = cpu_baseline_tile()
    if rank == 0:
        emit(line)
    if dist.is_initialized():
        dist.destroy_process_group()


# ---------------------------------------------------------------------------- our arm: other workloads
def run_workload(args):
    import numpy as np
    import torch
    import torch.distributed as dist

    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_icppw_nakanomi14_b200 as rap
    from paper_conf_icppw_nakanomi14_b200 import dist as rdist
    import workloads

    world, rank, local = dist_env()
    dev = torch.device("cuda", local % torch.cuda.device_count())
    torch.cuda.set_device(dev)
    init_dist(world, dev, force=args.workload == "dist_fused")
    stream = torch.cuda.current_stream()
    peak, peak_src = load_peaks()
    wl = args.workload
    barrier = (lambda: dist.barrier()) if world > 1 else (lambda: None)
    rmax = lambda v: reduce_over_ranks(v, world, dev, "max")

    # ---------------- workload setup
    if wl == "cfg4":
        rows = cols = 16384
        dt = torch.float64
    elif wl == "tile":
        rows = cols = 32
        dt = torch.float32
    elif wl in ("dist", "dist_fused"):
        rows, cols = 32768 // world, 32768
        dt = torch.float32
    else:
        rows = cols = 8192
        dt = torch.float32
    do_t = wl not in ("sweep", "trace")
    do_s = wl in ("cfg3", "sweep", "trace")
    layouts = (["raw", "pad", "xor", "ras", "rap"] if wl == "layouts"
               else ["rap16", "rap", "rap64"] if wl == "cfg4" and args.layout == "rap"     # T2b encodings beside the headline
               else [args.layout])
    eb = torch.empty((), dtype=dt).element_size()
    nbytes = 2 * rows * cols * eb                     # per rank per step
    x = workloads.random_bits(rows, cols, dt, seed=rank, device=dev) if do_t else None
    y = None
    dist_wl = wl in ("dist", "dist_fused")
    if do_t:
        y = torch.empty((rows, cols) if dist_wl else (cols, rows), dtype=dt, device=dev)
    work = {}
    fused = rdist.FusedTranspose((rows, cols), dt, layout=args.layout) if wl == "dist_fused" else None
    if fused is not None:
        y = fused.out
    S = args.sweep_trials
    hist = torch.zeros((5, 3, 33), dtype=torch.int64, device=dev)
    hstep = torch.zeros_like(hist)

    def step_transpose(lay):
        if wl == "dist_fused":
            fused(x)
            return 1                               # one fused transpose+exchange kernel (+ 2 barriers)
        if wl == "dist":
            rdist.transpose_sharded(x, layout=lay, seed=0, out=y, work=work)
            return 1 if world == 1 else 2          # local transpose (+ unpack)
        rap.transpose(x, layout=lay, seed=0, out=y)
        return 1

    # access traces (north star: "synthetic matrices and access traces"): 4096 warps of the paper's
    # pattern families, each evaluated under every step's trials and all five schemes
    trace_cells = workloads.trace_cells(4096, 32, seed=rank, device=dev) if wl == "trace" else None
    trace_hist = torch.zeros((5, 33), dtype=torch.int64, device=dev)
    TT = args.trace_trials                                 # trials per trace step

    def step_sweep(k):
        if wl == "trace":
            rap.congestion_trace(trace_cells, TT, seed=1, schemes=("raw", "ras", "rap", "pad", "xor"),
                                 first_trial=(k * world + rank) * TT, out=trace_hist)
            return 1
        # this rank's batch of the global trial sequence: step k covers trials
        # [k*S*world, (k+1)*S*world), rank r the r-th slice of it
        if world == 1:
            rap.congestion_sweep(S, seed=1, first_trial=k * S, out=hist, algo=args.sweep_algo)
            return 1
        # N > 1: this step's batch histogram, all-reduced (the sweep's one exchange), then added
        # to the run total (all-reducing the running total itself would count earlier steps again)
        hstep.zero_()
        rap.congestion_sweep(S, seed=1, first_trial=(k * world + rank) * S, out=hstep, algo=args.sweep_algo)
        all_reduce_hist(hstep, world)
        hist.add_(hstep)
        return 1

    soak_hist = torch.zeros_like(hist)

    def soak(lay, seconds):
        """Identical untimed steps (scratch histogram, far trial range) for `seconds`, in groups of
        16 between synchronisations; the same number of groups on every rank (soak_for: a step
        may hold the sharded transpose's all-to-all)."""
        def group(j):
            for i in range(16):
                k = 16 * j + i
                if do_t:
                    step_transpose(lay)
                if do_s and wl == "trace":
                    rap.congestion_trace(trace_cells, TT, seed=1, first_trial=(1 << 40) + k * TT,
                                         schemes=("raw", "ras", "rap", "pad", "xor"), out=torch.zeros_like(trace_hist))
                elif do_s:
                    rap.congestion_sweep(S, seed=1, first_trial=(1 << 40) + k * S, out=soak_hist, algo=args.sweep_algo)
        soak_for(seconds, group, world, dev)

    results = {}
    for lay in layouts:
        for k in range(args.warmup):
            if do_t:
                step_transpose(lay)
            if do_s:
                step_sweep(k)
        torch.cuda.synchronize()
        first_clocks = None
        for attempt in range(2):
            hist.zero_()
            launches, ev = 0, []
            barrier()
            torch.cuda.synchronize()
            with Clocks(dev.index) as clk:
                # the sampler runs over the timed steps and ~0.3 s of identical untimed steps on
                # each side, so every clock sample is taken under this workload
                soak(lay, 0.3)
                torch.cuda.synchronize()
                barrier()
                start = torch.cuda.Event(enable_timing=True)
                end = torch.cuda.Event(enable_timing=True)
                start.record(stream)
                for k in range(args.steps):
                    e = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
                    e[0].record(stream)
                    if do_t:
                        launches += step_transpose(lay)
                    e[1].record(stream)
                    e[2].record(stream)
                    if do_s:
                        launches += step_sweep(k)
                    e[3].record(stream)
                    ev.append(e)
                end.record(stream)
                torch.cuda.synchronize()
                barrier()
                soak(lay, 0.3)
                torch.cuda.synchronize()
            t_ms = [e[0].elapsed_time(e[1]) for e in ev]
            s_ms = [e[2].elapsed_time(e[3]) for e in ev]
            results[lay] = dict(total_ms=rmax(start.elapsed_time(end)), t_sum=rmax(sum(t_ms)), t_ms=t_ms,
                                s_sum=rmax(sum(s_ms)), s_ms=s_ms, clocks=clk.result, launches=launches)
            # a timed region that saw thermal / hardware slowdown, or SM clocks well below max with
            # no reason given, is measured once more (every rank agrees through the max)
            c = clk.result
            if attempt == 0 and rmax(1.0 if clocks_bad(c) else 0.0) > 0:
                first_clocks = c
                continue
            if first_clocks is not None:
                results[lay]["clocks"] = dict(c, remeasured=True, first_attempt=first_clocks)
            break

    lay = ("rap" if wl == "layouts" and "rap" in results
           else HEADLINE64 if wl == "cfg4" and HEADLINE64 in results else args.layout)
    r = results[lay]
    line = {"metric": METRIC, "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": r["total_ms"] / args.steps, "higher_is_better": True,
            "scaling": "strong" if dist_wl else "weak", "vs_baseline": None,
            "dtype": "u64" if eb == 8 else "u32", "data": "synthetic (seeded random bit patterns)"}
    if do_t:
        gbs = nbytes * world * args.steps / (r["t_sum"] * 1e-3) / 1e9
        kern_ms = r["t_sum"] / args.steps                # mean launch (the statistic of `value`)
        line.update(value=gbs, unit="GB/s")
        line["config"] = arm_config(args, world)
        assert line["config"]["layout"] == lay and line["config"]["algorithmic_bytes_per_step_per_rank"] == nbytes
        kkey = f"transpose_b{eb * 8}_{lay}"
        prof = load_profile(kkey) or {}
        if dist_wl and world > 1:
            nv = (world - 1) / world * (rows * cols * eb) / (kern_ms * 1e-3) / 1e9
            line["roofline"] = {"bound": "nvlink", "achieved": nv, "peak": NVLINK_GBS, "unit": "GB/s",
                                "frac": nv / NVLINK_GBS, "traffic": None,
                                "peak_source": "B200_PROFILING.md measured peer copy per direction",
                                "note": "bytes each rank sends over NVLink per step / step time"}
        else:
            line["roofline"] = hbm_roofline(nbytes, kern_ms, peak, peak_src, kkey)
        if wl in ("layouts", "cfg4") and len(results) > 1:
            line["layouts_gbs"] = {l: nbytes * world * args.steps / (v["t_sum"] * 1e-3) / 1e9
                                   for l, v in results.items()}
    if wl == "trace":
        evs = 4096 * TT * 5 * world * args.steps / (r["s_sum"] * 1e-3)
        th = trace_hist.cpu().numpy()
        c = np.arange(33)
        line.update(value=evs, unit="warp-evaluations/s",
                    config=arm_config(args, world))
        line["trace"] = {"E_by_scheme": {n: float((th[i] * c).sum() / th[i].sum())
                                         for i, n in enumerate(["raw", "ras", "rap", "pad", "xor"])},
                         "kernel_ms_median": statistics.median(r["s_ms"]),
                         # RAW / PAD / XOR use no random numbers: the kernel evaluates them once per
                         # (trace warp, block of 32 trials) and counts the result for every trial;
                         # the per-trial Monte-Carlo work is the RAS and RAP evaluations
                         "ras_rap_evaluations_per_s": evs * 2 / 5}
        line["roofline"] = trace_roofline(evs / world, r["clocks"])
    elif do_s:
        tps = S * world * args.steps / (r["s_sum"] * 1e-3)
        h = hist.cpu().numpy()
        c = np.arange(33)
        E = lambda a: float((a * c).sum() / a.sum())
        assert (h.sum(-1) == S * world * args.steps).all(), "histogram does not hold every timed trial once"
        line["sweep"] = {"trials_per_s": tps, "trials_per_step": S * world, "w": 32, "algo": args.sweep_algo,
                         "trials_in_histogram": int(h[0, 0].sum()),
                         "E_ras_stride": E(h[1, 1]), "E_rap_diagonal": E(h[2, 2]), "E_random": E(h[3, 2]),
                         "E_raw_malicious": E(h[4, 0]), "E_rap_stride": E(h[1, 2]),
                         "kernel_ms_mean": r["s_sum"] / args.steps,
                         "roofline": sweep_roofline(tps / world, r["clocks"])}
        if do_t and S <= 148 * 8 * 4 * 32:
            line["sweep"]["note"] = ("one batch of 32 trials per resident warp per step: a single wave, below the "
                                     "kernel's steady rate (launch ramp and tail); `--workload sweep` times 64 "
                                     "batches per warp per launch; the default workload sweeps 10^9 trials")
        if not do_t:
            line.update(value=tps, unit="trials/s",
                        config=arm_config(args, world))
            line["roofline"] = sweep_roofline(tps / world, r["clocks"])
    if do_t and do_s:
        t_share = r["t_sum"] / max(r["t_sum"] + r["s_sum"], 1e-9)
        line["kernel_time_share"] = {"transpose": t_share, "sweep": 1 - t_share}
        if t_share < 0.5:                       # the sweep dominates this step: report its roofline
            line["roofline_transpose"] = line["roofline"]
            line["roofline"] = line["sweep"]["roofline"]
    if wl == "tile":
        # latency case: the per-call time above includes the Python/ctypes launch path; replaying
        # 256 launches captured in one CUDA graph gives the device-side time per 32x32 transpose
        g = torch.cuda.CUDAGraph()
        cs = torch.cuda.Stream()
        cs.wait_stream(stream)
        with torch.cuda.stream(cs):
            rap.transpose(x, layout=lay, seed=0, out=y)
            torch.cuda.synchronize()
            with torch.cuda.graph(g, stream=cs):
                for _ in range(256):
                    rap.transpose(x, layout=lay, seed=0, out=y)
        g.replay()
        torch.cuda.synchronize()
        gs, ge = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        gs.record(stream)
        for _ in range(10):
            g.replay()
        ge.record(stream)
        torch.cuda.synchronize()
        us = gs.elapsed_time(ge) * 1e3 / (10 * 256)
        line["tile_latency"] = {"us_per_call_python": statistics.median(r["t_ms"]) * 1e3,
                                "us_per_transpose_cuda_graph": us,
                                "note": "2560 graph-replayed launches; includes the in-kernel Philox + "
                                        "Fisher-Yates of P (T0) and one 8 KiB tile"}
    line["clocks"] = r["clocks"]
    line["gpu_launches"] = int(reduce_over_ranks(r["launches"], world, dev, "sum"))

    # ---------------- e2e through the public API with pinned host buffers
    K = max(3, min(args.steps, 20))
    if not args.no_e2e and do_t and not dist_wl:
        # the end-to-end call: rap_transpose_host on pinned host buffers (H2D, transpose, D2H
        # pipelined over row bands on three streams -- PCIe both directions at once)
        hx = x.cpu().pin_memory()
        hy = torch.empty((cols, rows), dtype=dt).pin_memory()
        for _ in range(2):
            rap.transpose_host(hx, out=hy, layout=lay, seed=0, device=dev)
        barrier()
        st = torch.cuda.Event(enable_timing=True)
        en = torch.cuda.Event(enable_timing=True)
        st.record(stream)
        for _ in range(K):
            rap.transpose_host(hx, out=hy, layout=lay, seed=0, device=dev)
        en.record(stream)
        torch.cuda.synchronize()
        ms = rmax(st.elapsed_time(en)) / K
        bd = torch.int32 if eb == 4 else torch.int64
        rap.transpose(x, layout=lay, seed=0, out=y)
        assert torch.equal(hy.view(bd), y.cpu().view(bd)), "e2e result differs from the device result"
        line["e2e"] = {"value": nbytes * world / (ms * 1e-3) / 1e9, "unit": "GB/s",
                       "h2d_bytes_per_step": hx.numel() * eb * world, "d2h_bytes_per_step": hy.numel() * eb * world,
                       "ms_per_step": ms, "steps": K,
                       "note": "rap_transpose_host: pinned host matrix in, pinned host transpose out; "
                               "upload / RAP transpose / download of row bands (128 MiB workspace) overlapped"}
    elif not args.no_e2e and do_t:
        hx = x.cpu().pin_memory()
        hy = torch.empty(tuple(y.shape), dtype=dt).pin_memory()
        dx = torch.empty_like(x)

        def e2e_step():
            dx.copy_(hx, non_blocking=True)
            if wl == "dist_fused":
                fused(dx)
            else:
                rdist.transpose_sharded(dx, layout=lay, seed=0, out=y, work=work)
            hy.copy_(y, non_blocking=True)

        for _ in range(2):
            e2e_step()
        torch.cuda.synchronize()
        barrier()
        st = torch.cuda.Event(enable_timing=True)
        en = torch.cuda.Event(enable_timing=True)
        st.record(stream)
        for _ in range(K):
            e2e_step()
        en.record(stream)
        torch.cuda.synchronize()
        ms = rmax(st.elapsed_time(en)) / K
        bd = torch.int32 if eb == 4 else torch.int64
        assert torch.equal(hy.view(bd), y.cpu().view(bd)), "e2e result differs from the device result"
        line["e2e"] = {"value": nbytes * world / (ms * 1e-3) / 1e9, "unit": "GB/s",
                       "h2d_bytes_per_step": hx.numel() * eb * world, "d2h_bytes_per_step": hy.numel() * eb * world,
                       "ms_per_step": ms, "steps": K,
                       "note": "pinned host shard -> H2D -> sharded transpose (public API) -> D2H of the result"}
    elif not args.no_e2e and wl == "trace":
        # end to end: the step's access traces uploaded from pinned host memory, evaluated, and
        # the histogram read back
        hc = trace_cells.cpu().pin_memory()
        hh = torch.empty_like(trace_hist, device="cpu").pin_memory()
        st = torch.cuda.Event(enable_timing=True)
        en = torch.cuda.Event(enable_timing=True)
        st.record(stream)
        for k in range(K):
            trace_cells.copy_(hc, non_blocking=True)
            step_sweep(k)
            hh.copy_(trace_hist, non_blocking=True)
        en.record(stream)
        torch.cuda.synchronize()
        ms = rmax(st.elapsed_time(en)) / K
        line["e2e"] = {"value": 4096 * TT * 5 * world / (ms * 1e-3), "unit": "warp-evaluations/s",
                       "h2d_bytes_per_step": hc.numel() * 4 * world, "d2h_bytes_per_step": hh.numel() * 8 * world,
                       "ms_per_step": ms, "steps": K,
                       "note": "trace cells H2D from pinned memory + rap_congestion_trace + histogram D2H"}
    elif not args.no_e2e and do_s and wl != "trace":
        hh = torch.empty_like(hist, device="cpu").pin_memory()
        st = torch.cuda.Event(enable_timing=True)
        en = torch.cuda.Event(enable_timing=True)
        st.record(stream)
        for k in range(K):
            step_sweep(k)
            hh.copy_(hist, non_blocking=True)
        en.record(stream)
        torch.cuda.synchronize()
        ms = rmax(st.elapsed_time(en)) / K
        line["e2e"] = {"value": S * world / (ms * 1e-3), "unit": "trials/s", "h2d_bytes_per_step": 0,
                       "d2h_bytes_per_step": hh.numel() * 8, "ms_per_step": ms, "steps": K,
                       "note": "sweep batch through the public API + D2H of the histogram (inputs are counters)"}
    if rank == 0 and not args.no_cpu and world == 1:
        line["cpu_baseline"] = (cpu_baseline_transpose(rows, cols, dt) if do_t
                                else cpu_baseline_trace() if wl == "trace" else cpu_baseline_sweep())
        if do_s and do_t:
            line["sweep"]["cpu_baseline"] = cpu_baseline_sweep()
    if rank == 0:
        emit(line)
    if dist.is_initialized():
        dist.destroy_process_group()


def main():
    args = parse()
    route_native_stdout_to_stderr()
    if args.impl == "reference":
        return run_reference(args)
    if args.workload == "default":
        return run_default(args)
    return run_workload(args)


if __name__ == "__main__":
    main()
