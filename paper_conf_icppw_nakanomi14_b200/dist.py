"""Multi-GPU paths of the RAP hot path (one process per GPU, torch.distributed over NCCL).

Only two places shard:
  * congestion_sweep -- trials are independent (counter-based draws: trial n is a pure function
    of (seed, n)), so rank g sweeps the g-th contiguous slice of [first, first + N) and ONE
    all-reduce (SUM, int64) of the histogram combines them.  Integer sums are order-free, so
    the result is bit-identical to the one-GPU run and to the oracle for any world size.
  * transpose_sharded -- BASELINE cfg5: A (N x N) is row-block sharded, rank g holding rows
    gM..(g+1)M (M = N/G).  The local rap_transpose of the M x N shard yields N x M whose row
    block s is exactly the M x M block rank s needs; one all-to-all exchanges them and
    rap_unpack_blocks places the received blocks as rows gM..(g+1)M of A^T.
`local` hooks exist only so the exchange logic can be exercised with the gloo backend on CPU
(tests pass CPU stand-ins); by default every step is the CUDA library.
"""
from __future__ import annotations

import torch
import torch.distributed as dist

from . import congestion_sweep as _sweep
from . import transpose as _transpose
from . import transpose_to_peers as _to_peers
from . import unpack_blocks as _unpack


def _staged(t: torch.Tensor, group) -> bool:
    """gloo has no device collectives for these calls: stage CUDA tensors through host memory
    (the 1-GPU multi-process tests run gloo ranks that share one device)."""
    return t.is_cuda and dist.get_backend(group) != "nccl"


def all_reduce_sum(h: torch.Tensor, group=None) -> torch.Tensor:
    if _staged(h, group):
        hc = h.cpu()
        dist.all_reduce(hc, op=dist.ReduceOp.SUM, group=group)
        h.copy_(hc)
    else:
        dist.all_reduce(h, op=dist.ReduceOp.SUM, group=group)
    return h


def all_to_all(recv: torch.Tensor, send: torch.Tensor, group=None) -> torch.Tensor:
    if _staged(send, group):
        rc = torch.empty(recv.shape, dtype=recv.dtype)
        dist.all_to_all_single(rc, send.cpu(), group=group)
        recv.copy_(rc)
    else:
        dist.all_to_all_single(recv, send, group=group)
    return recv


def trial_slice(n_trials: int, rank: int, world: int, first_trial: int = 0):
    lo = first_trial + n_trials * rank // world
    hi = first_trial + n_trials * (rank + 1) // world
    return lo, hi - lo


def congestion_sweep(n_trials: int, seed: int, group=None, first_trial: int = 0, local=None,
                     out: torch.Tensor | None = None, **kw):
    """All-reduced histogram of [first_trial, first_trial + n_trials) swept across the group.

    The ranks sweep into a FRESH zeroed histogram, which is all-reduced and then added to `out`
    (if given): all-reducing a buffer that already holds counts would multiply them by the world
    size."""
    on = dist.is_initialized()
    rank, world = (dist.get_rank(group), dist.get_world_size(group)) if on else (0, 1)
    first, count = trial_slice(n_trials, rank, world, first_trial)
    fn = local if local is not None else _sweep
    h = fn(count, seed, first_trial=first, **kw)          # zero-initialised by the callee
    if world > 1:
        all_reduce_sum(h, group)
    if out is not None:
        out.add_(h)
        return out
    return h


def transpose_sharded(shard: torch.Tensor, group=None, layout: str = "rap", seed: int = 0,
                      out: torch.Tensor | None = None, local_transpose=None, local_unpack=None,
                      work: dict | None = None) -> torch.Tensor:
    """Rows gM..(g+1)M of A^T from rows gM..(g+1)M of A, for the whole group.

    shard: [M, N] with N = world * M.  Returns out: [M, N].  `work` may carry preallocated
    "send" / "recv" buffers ([N, M]) so repeated calls allocate nothing.
    """
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    M, N = shard.shape
    if N != world * M:
        raise ValueError(f"sharded transpose needs a square matrix: shard {M}x{N}, world {world}")
    tr = local_transpose if local_transpose is not None else (
        lambda x, o: _transpose(x, layout=layout, seed=seed, out=o))
    if out is None:
        out = torch.empty((M, N), dtype=shard.dtype, device=shard.device)
    if world == 1:                                    # nothing to exchange: transpose in place
        tr(shard, out)
        return out
    up = local_unpack if local_unpack is not None else (lambda r, o, G: _unpack(r, o, G))
    work = {} if work is None else work
    send = work.get("send")
    if send is None or send.shape != (N, M) or send.dtype != shard.dtype or send.device != shard.device:
        send = work["send"] = torch.empty((N, M), dtype=shard.dtype, device=shard.device)
        work["recv"] = torch.empty_like(send)
    recv = work["recv"]
    tr(shard, send)                                   # T1-T3: local RAP transpose, M x N -> N x M
    all_to_all(recv, send, group)                     # T4: M x M blocks, NCCL over NVLink
    up(recv, out, world)                              # T4: place the blocks
    return out


class FusedTranspose:
    """NEXT-2: the sharded transpose as ONE kernel per rank writing over NVLink into the peers'
    output shards.  No send/receive buffers, no all-to-all, no unpack: each element is read once
    from local HBM and written once, over NVLink when it belongs to another rank.

        ft = FusedTranspose((M, N), torch.float32, group)
        out = ft(shard)          # [M, N] tensor, rows rank*M.. of A^T, valid on return

    transport (how every rank's output buffer is mapped into every process):
      "symm"  torch symmetric memory; the two cross-rank barriers run on the device
              (default under NCCL);
      "ipc"   CUDA IPC handles of plain torch allocations (cudaIpcGetMemHandle /
              cudaIpcOpenMemHandle through torch's storage sharing), exchanged with
              all_gather_object; the barriers are device sync + dist.barrier() (default under
              gloo: works between processes that share one GPU, and between GPUs with P2P).
    """

    def __init__(self, shape, dtype, group=None, layout: str = "rap", seed: int = 0, transport: str | None = None):
        self.group = group if group is not None else dist.group.WORLD
        self.rank, self.world = dist.get_rank(self.group), dist.get_world_size(self.group)
        M, N = shape
        if N != self.world * M or M % 32:
            raise ValueError("fused transpose needs N = world * M and M a multiple of 32")
        dev = torch.device("cuda", torch.cuda.current_device())
        if transport is None:
            transport = "symm" if dist.get_backend(self.group) == "nccl" else "ipc"
        self.transport = transport
        if transport == "symm":
            from torch.distributed import _symmetric_memory as symm
            self.out = symm.empty((M, N), dtype=dtype, device=dev)
            self.handle = symm.rendezvous(self.out, self.group)
            self.ptrs = [int(p) for p in self.handle.buffer_ptrs]
        elif transport == "ipc":
            self.out = torch.empty((M, N), dtype=dtype, device=dev)
            mine = (self.out.untyped_storage()._share_cuda_(), self.out.storage_offset() * self.out.element_size())
            allh = [None] * self.world
            dist.all_gather_object(allh, mine, group=self.group)
            self._mapped = []                  # keeps the opened peer mappings alive
            self.ptrs = []
            for r, (h, off) in enumerate(allh):
                if r == self.rank:
                    self.ptrs.append(self.out.data_ptr())
                    continue
                st = torch.UntypedStorage._new_shared_cuda(*h)
                self._mapped.append(st)
                self.ptrs.append(st.data_ptr() + off)
        else:
            raise ValueError(f"unknown transport {transport!r}")
        self.layout, self.seed = layout, seed

    def _barrier(self):
        if self.transport == "symm":
            self.handle.barrier(channel=0)
        else:
            torch.cuda.current_stream().synchronize()
            dist.barrier(group=self.group)

    def __call__(self, shard: torch.Tensor) -> torch.Tensor:
        # every rank must be done reading its shard's previous contents before peers overwrite it
        self._barrier()
        _to_peers(shard, self.ptrs, self.rank, layout=self.layout, seed=self.seed)
        self._barrier()                     # all peers' stores into this shard have landed
        return self.out
