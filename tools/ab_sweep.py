"""Interleaved A/B of the cfg2 sweep (w = 32, 5 patterns x RAW/RAS/RAP) from several librap.so builds.

    python tools/ab_sweep.py --libs /tmp/a.so /tmp/b.so --trials 50000000 --rounds 7

Each arm sweeps --trials trials per launch (one launch between an event pair, after one warm-up
launch); arms interleaved per round; every arm's histogram must equal the first arm's.
"""
import argparse
import ctypes
import statistics

import torch


def load(path):
    L = ctypes.CDLL(path)
    u32, u64, vp = ctypes.c_uint32, ctypes.c_uint64, ctypes.c_void_p
    L.rap_congestion_sweep.argtypes = [u32, u32, u32, u64, u64, u64, vp, vp]
    L.rap_congestion_sweep.restype = ctypes.c_int
    return L


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--libs", nargs="+", required=True)
    ap.add_argument("--trials", type=int, default=50_000_000)
    ap.add_argument("--rounds", type=int, default=7)
    ap.add_argument("--w", type=int, default=32)
    a = ap.parse_args()
    libs = [(p, load(p)) for p in a.libs]
    st = ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
    h = torch.zeros((5, 3, a.w + 1), dtype=torch.int64, device="cuda")
    ref = None
    for p, L in libs:
        h.zero_()
        assert L.rap_congestion_sweep(a.w, 31, 7, 1, 0, 1_000_000, ctypes.c_void_p(h.data_ptr()), st) == 0
        torch.cuda.synchronize()
        if ref is None:
            ref = h.clone()
        assert torch.equal(h, ref), f"{p}: histogram differs"
    res = {p: [] for p, _ in libs}
    for r in range(a.rounds):
        for p, L in libs:
            L.rap_congestion_sweep(a.w, 31, 7, 1, 1 << 40, a.trials // 4, ctypes.c_void_p(h.data_ptr()), st)
            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s.record()
            L.rap_congestion_sweep(a.w, 31, 7, 1, r * a.trials, a.trials, ctypes.c_void_p(h.data_ptr()), st)
            e.record()
            torch.cuda.synchronize()
            res[p].append(a.trials / (s.elapsed_time(e) * 1e-3))
        print(f"round {r}: " + "  ".join(f"{k}={v[-1] / 1e9:.3f}G" for k, v in res.items()), flush=True)
    for k, v in res.items():
        print(f"{k:40s} median {statistics.median(v) / 1e9:.3f} G trials/s  min {min(v) / 1e9:.3f}  max {max(v) / 1e9:.3f}")


if __name__ == "__main__":
    main()
