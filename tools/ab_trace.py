"""Interleaved A/B of the w = 32 trace evaluator from several librap.so builds: 4096 synthetic
trace warps x --trials trials x 5 schemes per launch; every arm's histogram must equal the first's.
    python tools/ab_trace.py --libs /tmp/a.so /tmp/b.so"""
import argparse
import ctypes
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import workloads  # noqa: E402


def load(path):
    L = ctypes.CDLL(path)
    u32, u64, vp = ctypes.c_uint32, ctypes.c_uint64, ctypes.c_void_p
    L.rap_congestion_trace.argtypes = [u32, u64, vp, u32, u64, u64, u64, vp, vp]
    L.rap_congestion_trace.restype = ctypes.c_int
    return L


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--libs", nargs="+", required=True)
    ap.add_argument("--trials", type=int, default=2048)
    ap.add_argument("--rounds", type=int, default=7)
    a = ap.parse_args()
    cells = workloads.trace_cells(4096, 32, seed=0).cuda()
    h = torch.zeros((5, 33), dtype=torch.int64, device="cuda")
    st = ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
    libs = [(p, load(p)) for p in a.libs]
    call = lambda L, first: L.rap_congestion_trace(32, 4096, ctypes.c_void_p(cells.data_ptr()), 31, 1, first, a.trials,
                                                   ctypes.c_void_p(h.data_ptr()), st)
    ref = None
    for p, L in libs:
        h.zero_()
        assert call(L, 0) == 0
        torch.cuda.synchronize()
        ref = h.clone() if ref is None else ref
        assert torch.equal(h, ref), f"{p}: histogram differs"
    res = {p: [] for p, _ in libs}
    ev = 4096 * a.trials * 5
    for r in range(a.rounds):
        for p, L in libs:
            call(L, 1 << 30)
            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s.record()
            for k in range(5):
                call(L, (r * 5 + k) * a.trials)
            e.record()
            torch.cuda.synchronize()
            res[p].append(5 * ev / (s.elapsed_time(e) * 1e-3))
        print(f"round {r}: " + "  ".join(f"{k}={v[-1] / 1e9:.1f}G" for k, v in res.items()), flush=True)
    for k, v in res.items():
        print(f"{k:40s} median {statistics.median(v) / 1e9:.2f} G warp-evaluations/s  min {min(v) / 1e9:.2f}  max {max(v) / 1e9:.2f}")


if __name__ == "__main__":
    main()
