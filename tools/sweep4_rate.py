"""Throughput of the §VII w^4-array sweep (rap_congestion_sweep4, Table IV) at w = 16 and 32."""
import sys
import time

import torch

sys.path.insert(0, '.')
import __graft_entry__  # noqa: E402
__graft_entry__.build()
import paper_conf_icppw_nakanomi14_b200 as rap  # noqa: E402

for w, n in ((16, 1 << 22), (32, 1 << 22)):
    rap.congestion_sweep4(n // 16, seed=1, w=w)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    rap.congestion_sweep4(n, seed=1, w=w, first_trial=n)
    torch.cuda.synchronize()
    el = time.perf_counter() - t0
    print(f"sweep4 w={w}: {n / el / 1e6:8.1f} M trials/s (6 patterns x 5 schemes, {n} trials, {el * 1e3:.1f} ms)", flush=True)
