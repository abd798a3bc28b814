"""Where do the ~13 us between the cfg4 transpose's back-to-back launch time and its
event-bracketed time inside the default bench step go?  Mean per-launch time of the same
16384^2 float64 RAP transpose in different neighbourhoods (GPU box)."""
import statistics
import sys

import torch

sys.path.insert(0, '.')
import __graft_entry__  # noqa: E402
__graft_entry__.build()
import paper_conf_icppw_nakanomi14_b200 as rap  # noqa: E402
import workloads  # noqa: E402

x = workloads.random_bits(16384, 16384, torch.float64, seed=0, device="cuda")
y = torch.empty_like(x)
hist = torch.zeros((5, 3, 33), dtype=torch.int64, device="cuda")
small = torch.zeros(1 << 10, dtype=torch.float32, device="cuda")
NB = 2 * x.nbytes
K = 20


LAYOUT = sys.argv[1] if len(sys.argv) > 1 else "rap"


def bracketed(neigh):
    evs = []
    for k in range(K + 3):
        e = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
        e[0].record()
        rap.transpose(x, layout=LAYOUT, out=y)
        e[1].record()
        if neigh == "sweep":
            rap.congestion_sweep(50_000_000, seed=1, first_trial=k * 50_000_000, out=hist)
        elif neigh == "sweep_small":
            rap.congestion_sweep(151552, seed=1, first_trial=k * 151552, out=hist)
        elif neigh == "tiny":
            small.add_(1.0)
        if k >= 3:
            evs.append(e)
    torch.cuda.synchronize()
    return statistics.mean(e[0].elapsed_time(e[1]) for e in evs) * 1e-3


def back_to_back():
    for _ in range(3):
        rap.transpose(x, layout=LAYOUT, out=y)
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    for _ in range(K):
        rap.transpose(x, layout=LAYOUT, out=y)
    e.record()
    torch.cuda.synchronize()
    return s.elapsed_time(e) * 1e-3 / K


print("layout", LAYOUT)
for rnd in range(3):
    r = {"back_to_back": back_to_back(), "bracketed_alone": bracketed(None), "bracketed_tiny": bracketed("tiny"),
         "bracketed_sweep_small": bracketed("sweep_small"), "bracketed_sweep_5e7": bracketed("sweep")}
    print("  ".join(f"{k} {v * 1e6:.1f} us ({NB / v / 1e9:.0f} GB/s)" for k, v in r.items()), flush=True)
