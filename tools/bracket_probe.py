"""Why is the 8192^2 transpose 4-5 us slower inside bench.py's step than back to back in a CUDA
graph?  Per-launch event times of the same RAP transpose in different neighbourhoods."""
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
hist = torch.zeros((5, 3, 33), dtype=torch.int64, device="cuda")
small = torch.zeros(1 << 20, dtype=torch.float32, device="cuda")
NB = 2 * x.nbytes


def run(neigh, steps=40):
    evs = []
    for k in range(steps + 3):
        e = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
        e[0].record()
        rap.transpose(x, layout="rap", out=y)
        e[1].record()
        if neigh == "sweep":
            rap.congestion_sweep(151552, seed=1, first_trial=k * 151552, out=hist)
        elif neigh == "tiny":
            small.add_(1.0)
        elif neigh == "bigwrite":                    # 256 MiB of unrelated writes (evicts L2)
            y.fill_(0)
        if k >= 3:
            evs.append(e)
    torch.cuda.synchronize()
    return statistics.median(e[0].elapsed_time(e[1]) for e in evs) * 1e-3


for rnd in range(2):
    for neigh in ("none", "tiny", "sweep", "bigwrite"):
        t = run(neigh)
        print(f"after {neigh:9s}: {t * 1e6:7.1f} us  {NB / t / 1e9:7.1f} GB/s", flush=True)
