"""Throughput of the congestion sweep for w = 16, 32 (warp kernels) and 64, 128, 256 (sweep_wide)."""
import sys
import time

import torch

sys.path.insert(0, '.')
import __graft_entry__  # noqa: E402
__graft_entry__.build()
import paper_conf_icppw_nakanomi14_b200 as rap  # noqa: E402

for w, n in ((16, 1 << 24), (32, 1 << 26), (64, 1 << 21), (128, 1 << 20), (256, 1 << 19)):
    h = rap.congestion_sweep(n // 16, seed=1, w=w)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    h = rap.congestion_sweep(n, seed=1, w=w, first_trial=n)
    torch.cuda.synchronize()
    el = time.perf_counter() - t0
    print(f"w={w:3d}: {n / el / 1e6:9.1f} M trials/s ({n} trials, {el * 1e3:.1f} ms)", flush=True)
