"""Does access granularity explain fp64 (0.94-0.98 of copy) vs fp32 (0.87)?  Same 256 MiB buffer:
fp32 8192x8192 RAP (128 B row segments), the same bytes as an 8192x4096 fp64 matrix under the
two-plane RAP and RAP-16 kernels (256 B row segments), and cudaMemcpy; interleaved rounds."""
import statistics
import sys

import torch

sys.path.insert(0, '.')
import __graft_entry__  # noqa: E402
__graft_entry__.build()
import paper_conf_icppw_nakanomi14_b200 as rap  # noqa: E402
import workloads  # noqa: E402

x = workloads.random_bits(8192, 8192, torch.float32, seed=0, device="cuda")
y = torch.empty_like(x)
x64 = x.view(torch.float64)            # 8192 x 4096
y64 = torch.empty((4096, 8192), dtype=torch.float64, device="cuda")
big = workloads.random_bits(16384, 16384, torch.float32, seed=1, device="cuda")     # 1 GiB
ybig = torch.empty_like(big)
cases = {
    "fp32 8192x8192 rap": (lambda: rap.transpose(x, layout="rap", out=y), 2 * x.nbytes),
    "fp64 8192x4096 rap (two planes)": (lambda: rap.transpose(x64, layout="rap", out=y64), 2 * x.nbytes),
    "fp64 8192x4096 rap16": (lambda: rap.transpose(x64, layout="rap16", out=y64), 2 * x.nbytes),
    "memcpy 256 MiB": (lambda: y.copy_(x), 2 * x.nbytes),
    "fp32 16384x16384 rap (1 GiB)": (lambda: rap.transpose(big, layout="rap", out=ybig), 2 * big.nbytes),
    "memcpy 1 GiB": (lambda: ybig.copy_(big), 2 * big.nbytes),
}
res = {k: [] for k in cases}
ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
for rnd in range(7):
    for k, (fn, nb) in cases.items():
        for _ in range(3):
            fn()
        ts = []
        for _ in range(10):
            ev[0].record(); fn(); ev[1].record(); torch.cuda.synchronize()
            ts.append(ev[0].elapsed_time(ev[1]))
        res[k].append(statistics.median(ts))
for k, (fn, nb) in cases.items():
    t = statistics.median(res[k])
    print(f"{k:36s} {nb / t / 1e6:8.1f} GB/s  {t * 1e3:8.1f} us")
