"""RAP transpose throughput vs matrix size and element width (GPU box): is the fp32 / fp64 gap a
per-launch fixed cost (vanishing with size) or a per-byte difference?  Back-to-back launches."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import __graft_entry__  # noqa: E402
__graft_entry__.build()
import paper_conf_icppw_nakanomi14_b200 as rap  # noqa: E402
import workloads  # noqa: E402

PEAK = 6548.2
for dt, sizes in ((torch.float32, (4096, 8192, 11584, 16384, 23168, 32768)),
                  (torch.float64, (4096, 5792, 8192, 11584, 16384, 23168))):
    for n in sizes:
        x = workloads.random_bits(n, n, dt, seed=0, device="cuda")
        y = torch.empty_like(x)
        nb = 2 * x.numel() * x.element_size()
        res = []
        for r in range(5):
            for _ in range(3):
                rap.transpose(x, layout="rap", out=y)
            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            k = max(5, int(2e10 / nb))
            s.record()
            for _ in range(k):
                rap.transpose(x, layout="rap", out=y)
            e.record()
            torch.cuda.synchronize()
            res.append(s.elapsed_time(e) / k)
        ms = sorted(res)[len(res) // 2]
        print(f"{str(dt)[6:]:8s} {n:6d}^2  {nb / 2**20:8.0f} MiB  {ms * 1e3:9.1f} us  {nb / (ms * 1e-3) / 1e9:7.0f} GB/s  "
              f"{nb / (ms * 1e-3) / 1e9 / PEAK:.3f}", flush=True)
        del x, y
        torch.cuda.empty_cache()
