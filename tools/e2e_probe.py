import sys, time, torch
sys.path.insert(0, '.')
import __graft_entry__; __graft_entry__.build()
import paper_conf_icppw_nakanomi14_b200 as rap, workloads
for (r, c, dt) in ((8192, 8192, torch.float32), (16384, 16384, torch.float64)):
    x = workloads.random_bits(r, c, dt, seed=0).pin_memory()
    y = torch.empty((c, r), dtype=dt).pin_memory()
    nbytes = 2 * x.numel() * x.element_size()
    for ws in (16 << 20, 32 << 20, 64 << 20, 128 << 20, 256 << 20):
        rap.transpose_host(x, out=y, workspace_bytes=ws)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(5):
            rap.transpose_host(x, out=y, workspace_bytes=ws)
        el = (time.perf_counter() - t0) / 5
        print(r, c, dt, 'ws MiB', ws >> 20, f'{nbytes / el / 1e9:.1f} GB/s', f'{el*1e3:.2f} ms')
    t0 = time.perf_counter()
    d = x.cuda(); torch.cuda.synchronize(); t1 = time.perf_counter(); h = d.cpu(); t2 = time.perf_counter()
    print('plain H2D', x.nbytes / (t1 - t0) / 1e9, 'D2H (pageable)', x.nbytes / (t2 - t1) / 1e9)
    dd = torch.empty_like(d); torch.cuda.synchronize(); t0 = time.perf_counter(); dd.copy_(x, non_blocking=True); torch.cuda.synchronize(); t1 = time.perf_counter()
    y.copy_(d, non_blocking=True); torch.cuda.synchronize(); t2 = time.perf_counter()
    print('pinned H2D', x.nbytes / (t1 - t0) / 1e9, 'pinned D2H', x.nbytes / (t2 - t1) / 1e9)
