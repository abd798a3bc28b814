"""Small invocations of every librap kernel, for compute-sanitizer (memcheck / racecheck /
synccheck / initcheck) runs:  compute-sanitizer --tool racecheck python tools/sanitize.py"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import __graft_entry__  # noqa: E402

__graft_entry__.build()
import paper_conf_icppw_nakanomi14_b200 as rap  # noqa: E402
import workloads  # noqa: E402

dev = torch.device("cuda", 0)
for dt in (torch.float32, torch.float64):
    for (r, c) in ((33, 65), (96, 200), (256, 256)):
        x = workloads.random_bits(r, c, dt, seed=1).to(dev)
        for lay in rap.LAYOUTS:
            if lay in ("rap16", "rap64") and dt == torch.float32:
                continue
            y = rap.transpose(x, layout=lay, seed=3)
            assert torch.equal(y.cpu().view(torch.int32 if dt == torch.float32 else torch.int64),
                               x.cpu().t().contiguous().view(torch.int32 if dt == torch.float32 else torch.int64))
    xs = workloads.random_bits(100, 64, dt, seed=2).to(dev)[:, 1:60]
    rap.transpose(xs, layout="rap")
rap.perm_gen_batch(seed=1, count=100, w=32)
rap.perm_gen_batch(seed=1, count=10, w=7)
rap.congestion_sweep(5000, seed=1)
rap.congestion_sweep(5000, seed=1, schemes=("raw", "ras", "rap", "pad", "xor"))
rap.congestion_sweep(3000, seed=1, w=7, schemes=("raw", "ras", "rap", "pad"))
rap.congestion_sweep(3000, seed=1, w=16)
rap.congestion_sweep(300, seed=1, w=64)
rap.congestion_sweep(200, seed=1, w=100, schemes=("raw", "ras", "rap", "pad"))
rap.congestion_sweep(100, seed=1, w=256, schemes=("raw", "ras", "rap", "pad", "xor"))
rap.congestion_sweep(2000, seed=1, algo="match")
rap.congestion_sweep4(2000, seed=1, w=16)
cells = workloads.trace_cells(20, 32, seed=1).to(dev)
rap.congestion_trace(cells, 10, seed=1, schemes=("raw", "ras", "rap", "pad", "xor"))
cells2 = workloads.trace_cells(131, 32, seed=2)
cells2[7, 3] = 5000                                   # invalid trace warp -> bin 0
rap.congestion_trace(cells2.to(dev), 70, seed=1, schemes=("ras", "xor"), first_trial=33)
cells3 = workloads.trace_cells(40, 8, seed=3)
cells3[2, 1] = 64                                     # w = 8: invalid trace warp
rap.congestion_trace(cells3.to(dev), 37, seed=1, schemes=("raw", "ras", "rap", "pad", "xor"))
t = lambda a: torch.from_numpy(np.asarray(a, dtype=np.int32)).to(dev)
rr = np.random.default_rng(0).integers(0, 32, (50, 32))
rap.congestion(t(rr), t(rr[::-1].copy()), "rap", shift=t(np.stack([np.random.default_rng(k).permutation(32) for k in range(50)])))
for alg in ("crsw", "srcw", "drdw"):
    for sch in ("raw", "ras", "rap"):
        rap.smem_transpose_bench(alg, sch, 4, 1, 2, 3)
idx = workloads.tile_gather_patterns(seed=1)["random"]
for lay in ("raw", "pad", "xor", "ras", "rap"):
    rap.smem_gather_bench(torch.from_numpy(idx.view(np.int16)).to(dev), lay, 1, 2, 3)
G, M = 2, 64
A = workloads.random_bits(G * M, G * M, torch.float32, seed=5).to(dev)
outs = [torch.zeros((M, G * M), device=dev) for _ in range(G)]
for g in range(G):
    rap.transpose_to_peers(A[g * M:(g + 1) * M], [o.data_ptr() for o in outs], g)
recv = workloads.random_bits(G * M, M, torch.float32, seed=6).to(dev)
rap.unpack_blocks(recv, torch.empty((M, G * M), device=dev), G)
h = workloads.random_bits(300, 200, torch.float32, seed=7).pin_memory()
rap.transpose_host(h, workspace_bytes=1 << 20)
torch.cuda.synchronize()
print("sanitize workload done")
