"""Fixed vs per-byte cost of one transpose launch: t(rows) for rows x 8192 fp32 matrices, fitted
t = a + bytes / B (least squares), for the library kernel and for cudaMemcpy of the same bytes.
Each point is a CUDA graph of 10 back-to-back launches (no host launch latency in the window)."""
import statistics
import sys

import numpy as np
import torch

sys.path.insert(0, '.')
import __graft_entry__  # noqa: E402
__graft_entry__.build()
import paper_conf_icppw_nakanomi14_b200 as rap  # noqa: E402
import workloads  # noqa: E402

ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]


def med(fn, reps=15, per_graph=10):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for _ in range(per_graph):
            fn()
    g.replay()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        ev[0].record(); g.replay(); ev[1].record(); torch.cuda.synchronize()
        ts.append(ev[0].elapsed_time(ev[1]) / per_graph)
    return statistics.median(ts) * 1e-3


rows_list = [1024, 2048, 4096, 8192, 16384, 32768]
X = workloads.random_bits(32768, 8192, torch.float32, seed=0, device="cuda")
Y = torch.empty((8192, 32768), dtype=torch.float32, device="cuda")
for name in ("rap", "raw", "memcpy"):
    ts, bs = [], []
    for r in rows_list:
        x = X[:r]
        y = Y[:, :r] if name != "memcpy" else Y.view(-1)[: r * 8192].view(r, 8192)
        if name == "memcpy":
            fn = lambda: y.copy_(x)
        else:
            yy = torch.empty((8192, r), dtype=torch.float32, device="cuda")
            fn = lambda: rap.transpose(x, layout=name, out=yy)
        t = statistics.median([med(fn) for _ in range(3)])
        ts.append(t); bs.append(2 * x.nbytes)
    A = np.vstack([np.ones(len(bs)), np.array(bs)]).T
    (a, inv_b), *_ = np.linalg.lstsq(A, np.array(ts), rcond=None)
    print(f"{name:7s} fixed {a * 1e6:6.2f} us, asymptotic {1 / inv_b / 1e9:7.1f} GB/s;  " +
          "  ".join(f"{r}:{b / t / 1e9:.0f}" for r, b, t in zip(rows_list, bs, ts)), flush=True)
