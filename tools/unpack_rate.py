"""Bandwidth of rap_unpack_blocks (T4, the NCCL path's block placement after the all-to-all) for
cfg5's per-rank shapes: G blocks of M x M fp32 (N = 32768, M = N / G) into an M x N output."""
import statistics
import sys

import torch

sys.path.insert(0, '.')
import __graft_entry__  # noqa: E402
__graft_entry__.build()
import paper_conf_icppw_nakanomi14_b200 as rap  # noqa: E402

ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
for G in (2, 4, 8):
    N = 32768
    M = N // G
    recv = torch.empty((G * M, M), dtype=torch.float32, device="cuda").random_()
    out = torch.empty((M, N), dtype=torch.float32, device="cuda")
    for _ in range(3):
        rap.unpack_blocks(recv, out, G)
    ts = []
    for _ in range(20):
        ev[0].record(); rap.unpack_blocks(recv, out, G); ev[1].record(); torch.cuda.synchronize()
        ts.append(ev[0].elapsed_time(ev[1]) * 1e-3)
    t = statistics.median(ts)
    ts2 = []
    for _ in range(20):
        ev[0].record(); out.view(-1).copy_(recv.view(-1)); ev[1].record(); torch.cuda.synchronize()
        ts2.append(ev[0].elapsed_time(ev[1]) * 1e-3)
    t2 = statistics.median(ts2)
    print(f"G={G}: unpack {2 * recv.nbytes / t / 1e9:7.1f} GB/s ({t * 1e6:.1f} us); plain copy of the same bytes "
          f"{2 * recv.nbytes / t2 / 1e9:7.1f} GB/s", flush=True)
