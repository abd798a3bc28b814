"""Size-matched copy ceiling (GPU box): torch's device-to-device copy_ of the same bytes as each
bench transpose (cfg3: 256 MiB in + 256 MiB out, cfg4: 2 GiB + 2 GiB, cfg5: 4 GiB + 4 GiB) and
the RAP transposes beside it, back to back between one event pair, interleaved rounds.

MEASURED_PEAKS.json's hbm_gbs is one copy at 2 GiB; a smaller copy pays the same ramp-up /
tail / launch costs a transpose of that size pays, so this says how much of the cfg3 deficit is
the size rather than the kernel."""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import __graft_entry__  # noqa: E402
__graft_entry__.build()
import paper_conf_icppw_nakanomi14_b200 as rap  # noqa: E402
import workloads  # noqa: E402

CASES = [("cfg3 8192^2 f32", 8192, torch.float32, ["rap", "pad", "xor"]),
         ("cfg4 16384^2 f64", 16384, torch.float64, ["rap64", "rap", "rap16"]),
         ("cfg5 32768^2 f32", 32768, torch.float32, ["rap"])]


def timed(fn, k):
    for _ in range(3):
        fn()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    for _ in range(k):
        fn()
    e.record()
    torch.cuda.synchronize()
    return s.elapsed_time(e) / k


for name, n, dt, lays in CASES:
    x = workloads.random_bits(n, n, dt, seed=0, device="cuda")
    y = torch.empty_like(x)
    nb = 2 * x.numel() * x.element_size()
    k = max(10, int(2e10 / nb))
    arms = {"copy_": lambda: y.copy_(x)}
    for lay in lays:
        arms[lay] = (lambda l: lambda: rap.transpose(x, layout=l, seed=0, out=y))(lay)
    res = {a: [] for a in arms}
    for r in range(7):
        for a, fn in arms.items():
            res[a].append(nb / (timed(fn, k) * 1e-3) / 1e9)
    cp = statistics.median(res["copy_"])
    print(f"{name}: {nb / 2**20:.0f} MiB per launch, {k} launches per event pair, medians of 7 interleaved rounds")
    for a, v in res.items():
        m = statistics.median(v)
        print(f"  {a:8s} {m:8.1f} GB/s  (min {min(v):.1f}, max {max(v):.1f})  {m / cp:.3f} of the size-matched copy_",
              flush=True)
    del x, y
    torch.cuda.empty_cache()
