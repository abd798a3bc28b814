"""e2e probe (GPU box): rap_transpose_host throughput vs workspace size, and the PCIe ceiling it
runs against -- one-way pinned H2D / D2H and both directions at once on two streams."""
import sys
import time

import torch

sys.path.insert(0, '.')
import __graft_entry__  # noqa: E402
__graft_entry__.build()
import paper_conf_icppw_nakanomi14_b200 as rap  # noqa: E402
import workloads  # noqa: E402


def t_of(fn, reps=5):
    fn()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(reps):
        fn()
    torch.cuda.synchronize()
    return (time.perf_counter() - t0) / reps


for (r, c, dt) in ((8192, 8192, torch.float32), (16384, 16384, torch.float64)):
    x = workloads.random_bits(r, c, dt, seed=0).pin_memory()
    y = torch.empty((c, r), dtype=dt).pin_memory()
    nbytes = 2 * x.numel() * x.element_size()
    for ws in (64 << 20, 128 << 20, 256 << 20, 512 << 20, 1024 << 20):
        el = t_of(lambda: rap.transpose_host(x, out=y, workspace_bytes=ws))
        print(r, c, str(dt)[6:], 'ws MiB', ws >> 20, f'{nbytes / el / 1e9:.1f} GB/s', f'{el * 1e3:.2f} ms', flush=True)
    d = x.cuda()
    d2 = torch.empty_like(d)
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    h2d = t_of(lambda: d2.copy_(x, non_blocking=True))
    d2h = t_of(lambda: y.view(-1).copy_(d.view(-1), non_blocking=True))

    def both():
        with torch.cuda.stream(s1):
            d2.copy_(x, non_blocking=True)
        with torch.cuda.stream(s2):
            y.view(-1).copy_(d.view(-1), non_blocking=True)
    bi = t_of(both)
    nb = x.nbytes
    print(f'pinned H2D {nb / h2d / 1e9:.1f} GB/s, D2H {nb / d2h / 1e9:.1f} GB/s, both at once {2 * nb / bi / 1e9:.1f} GB/s '
          f'({bi * 1e3:.2f} ms for {nb >> 20} MiB each way)', flush=True)
