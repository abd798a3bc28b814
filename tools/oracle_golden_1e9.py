"""Write the oracle's full-size cfg2 histograms (w = 32, 10^9 trials, seeds 1, 2, 3) as golden files.

BASELINE.json cfg2: "DMM congestion sweep w=32: contiguous/stride/random/malicious warp patterns,
10^9 Philox permutations"; the north star asks the GPU sweep to match the oracle bit for bit per
seed at that size.  The oracle takes ~30 min per seed on 8 host cores, far too long for a test,
so this committed script runs it once (it calls only `oracle/`) and stores
tests/golden/sweep_w32_1e9_seed<s>.txt; tests/test_gpu_parity.py compares the GPU against them.

    python tools/oracle_golden_1e9.py [--seeds 1 2 3] [--chunk 50000000] [--threads N]

Chunks are accumulated (the oracle sweep is additive over trial ranges, pinned by
tests/test_oracle_pins.py::test_sweep_is_additive_over_trial_ranges) so progress survives in a
partial file (<name>.partial) and the run can be resumed.
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402  (test infrastructure; this script only feeds tests/golden)

PATTERNS = ["contiguous", "stride", "diagonal", "random", "malicious"]
SCHEMES = ["raw", "ras", "rap"]
N = 10 ** 9


def golden_path(seed: int) -> str:
    return os.path.join(ROOT, "tests", "golden", f"sweep_w32_1e9_seed{seed}.txt")


def write(path: str, seed: int, done: int, h: np.ndarray, seconds: float, threads: int) -> None:
    with open(path, "w") as f:
        f.write("# cfg2 congestion sweep, w = 32, oracle/rap_oracle.c (tools/oracle_golden_1e9.py)\n")
        f.write(f"# seed {seed}, trials [0, {done}), patterns {' '.join(PATTERNS)}, schemes {' '.join(SCHEMES)}\n")
        f.write(f"# {json.dumps({'seed': seed, 'first_trial': 0, 'n_trials': done, 'oracle_seconds': round(seconds, 1), 'threads': threads})}\n")
        f.write("# one line per (pattern, scheme): pattern scheme h[0] h[1] ... h[32]\n")
        for p, pn in enumerate(PATTERNS):
            for s, sn in enumerate(SCHEMES):
                f.write(f"{pn} {sn} " + " ".join(str(int(v)) for v in h[p, s]) + "\n")


def read(path: str):
    meta, h = None, np.zeros((5, 3, 33), dtype=np.uint64)
    for ln in open(path):
        if ln.startswith("# {"):
            meta = json.loads(ln[2:])
        elif not ln.startswith("#") and ln.strip():
            f = ln.split()
            h[PATTERNS.index(f[0]), SCHEMES.index(f[1])] = np.array([int(v) for v in f[2:]], dtype=np.uint64)
    return meta, h


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--seeds", type=int, nargs="+", default=[1, 2, 3])
    ap.add_argument("--chunk", type=int, default=50_000_000)
    ap.add_argument("--threads", type=int, default=None)
    a = ap.parse_args()
    th = a.threads or oracle.max_threads()
    for seed in a.seeds:
        out = golden_path(seed)
        part = out + ".partial"
        if os.path.exists(out):
            print(f"seed {seed}: {out} exists", flush=True)
            continue
        done, h, spent = 0, np.zeros((5, 3, 33), dtype=np.uint64), 0.0
        if os.path.exists(part):
            meta, h = read(part)
            done, spent = meta["n_trials"], meta["oracle_seconds"]
        while done < N:
            n = min(a.chunk, N - done)
            t0 = time.time()
            h += oracle.sweep(32, PATTERNS, SCHEMES, seed, done, n, threads=th)
            spent += time.time() - t0
            done += n
            write(part, seed, done, h, spent, th)
            print(f"seed {seed}: {done / N:.0%} ({spent:.0f} s)", flush=True)
        assert (h.sum(-1) == N).all()
        os.replace(part, out)


if __name__ == "__main__":
    main()
