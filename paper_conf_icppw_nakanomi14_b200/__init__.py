"""RAP (Random Address Permute-Shift, Nakano-Matsumae-Ito, ICPPW 2014) on B200.

Thin Python binding over ``librap.so`` (C ABI: ``include/rap.h``).  Every step of the hot
path runs in the library's sm_100a kernels; this module only marshals torch tensors (device
memory), the current CUDA stream and the enums.  There is no CPU fallback: calling with a
CPU tensor, or without the built library, raises.

Functions keep the C names without the ``rap_`` prefix:
  hot path      perm_gen (host), perm_gen_batch, transpose, congestion, congestion_sweep (+ algo), congestion_trace
  host / multi  transpose_host (host-to-host pipeline), unpack_blocks, transpose_to_peers
                (the multi-GPU drivers are in ``dist``)
  paper §VI/VII smem_transpose_bench (Table III), congestion_sweep4 (§VII, Table IV),
                smem_gather_bench (data-dependent access under a layout)
"""
from __future__ import annotations

import contextlib
import ctypes
import os

import torch

from . import build as _build

__all__ = ["perm_gen", "perm_gen_batch", "transpose", "transpose_host", "transpose_to_peers", "congestion", "congestion_sweep",
           "congestion_trace", "unpack_blocks", "smem_transpose_bench", "congestion_sweep4", "smem_gather_bench",
           "LAYOUTS", "SCHEMES", "PATTERNS", "SWEEP_ALGOS", "SMEM_ALGORITHMS", "SCHEMES4", "PATTERNS4",
           "RapError", "lib", "library_path"]

LAYOUTS = {"raw": 0, "pad": 1, "xor": 2, "ras": 3, "rap": 4, "rap16": 5, "rap64": 6}   # rap16/rap64: 8-byte only
SCHEMES = {"raw": 0, "ras": 1, "rap": 2, "pad": 3, "xor": 4}
SWEEP_ALGOS = {"default": 0, "match": 1}
PATTERNS = {"contiguous": 0, "stride": 1, "diagonal": 2, "random": 3, "malicious": 4}
SMEM_ALGORITHMS = {"crsw": 0, "srcw": 1, "drdw": 2}
SCHEMES4 = {"raw": 0, "ras": 1, "1p": 2, "r1p": 3, "3p": 4}
PATTERNS4 = {"contiguous": 0, "stride1": 1, "stride2": 2, "stride3": 3, "random": 4, "malicious": 5}
STATUS = {0: "RAP_OK", 1: "RAP_ERR_INVALID_ARG", 2: "RAP_ERR_UNSUPPORTED", 3: "RAP_ERR_ALIAS",
          4: "RAP_ERR_CUDA"}


class RapError(RuntimeError):
    def __init__(self, status: int, what: str):
        super().__init__(f"{what}: {STATUS.get(status, status)}")
        self.status = status


_lib = None


def library_path() -> str:
    return _build.LIB


def lib():
    """Load librap.so (built in-tree by ``__graft_entry__.build()``); raise if it is missing."""
    global _lib
    if _lib is None:
        path = _build.LIB
        if not os.path.exists(path):
            raise ImportError(f"{path} is missing: run `python -c 'import __graft_entry__ as g; "
                              "g.build()'` (no CPU fallback exists)")
        L = ctypes.CDLL(path)
        u8p, u32p, u64p, vp = (ctypes.c_void_p,) * 4
        i32, u32, u64, i64 = ctypes.c_int, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int64
        L.rap_abi_version.restype = i32
        L.rap_status_str.argtypes = [i32]
        L.rap_status_str.restype = ctypes.c_char_p
        L.rap_perm_gen.argtypes = [u64, u64, u32, ctypes.POINTER(u32)]
        L.rap_perm_gen_batch.argtypes = [u64, u64, u64, u32, u8p, vp]
        L.rap_transpose.argtypes = [vp, vp, i64, i64, i64, i64, u32, i32, u64, vp]
        L.rap_congestion.argtypes = [u32, u64, u32p, u32p, i32, u32p, u32p, vp]
        L.rap_congestion_sweep.argtypes = [u32, u32, u32, u64, u64, u64, u64p, vp]
        L.rap_congestion_sweep_algo.argtypes = [u32, u32, u32, u64, u64, u64, u64p, u32, vp]
        L.rap_congestion_trace.argtypes = [u32, u64, u32p, u32, u64, u64, u64, u64p, vp]
        L.rap_unpack_blocks.argtypes = [vp, vp, i64, i64, i64, u32, vp]
        L.rap_congestion_sweep4.argtypes = [u32, u32, u32, u64, u64, u64, u64p, vp]
        L.rap_transpose_host.argtypes = [vp, vp, i64, i64, i64, i64, u32, i32, u64, vp, ctypes.c_size_t, vp]
        L.rap_smem_gather_bench.argtypes = [vp, i32, u64, u32, u32, u32p, u64p, vp]
        L.rap_smem_transpose_bench.argtypes = [u32, i32, u32, u64, u32, u32, u32p, u64p, vp]
        L.rap_transpose_to_peers.argtypes = [vp, i64, i64, i64, ctypes.POINTER(ctypes.c_void_p), u32, u32, i64,
                                             u32, i32, u64, vp]
        for f in ("rap_perm_gen", "rap_perm_gen_batch", "rap_transpose", "rap_congestion", "rap_congestion_sweep",
                  "rap_congestion_sweep_algo", "rap_congestion_trace", "rap_unpack_blocks",
                  "rap_smem_transpose_bench", "rap_transpose_to_peers", "rap_congestion_sweep4",
                  "rap_smem_gather_bench", "rap_transpose_host"):
            getattr(L, f).restype = i32
        if L.rap_abi_version() != 2:
            raise ImportError("librap.so ABI version mismatch")
        _lib = L
    return _lib


_raw_stream = getattr(torch._C, "_cuda_getCurrentRawStream", None)


def _stream(t: torch.Tensor):
    """The current CUDA stream of t's device, as the cudaStream_t handle (cheap raw lookup)."""
    if _raw_stream is not None:
        return ctypes.c_void_p(_raw_stream(t.device.index if t.device.index is not None
                                           else torch.cuda.current_device()))
    return ctypes.c_void_p(torch.cuda.current_stream(t.device).cuda_stream)


def _on(dev: torch.device):
    """Make `dev` current for the C call (no-op, and no context-manager cost, when it already is)."""
    if dev.index is None or dev.index == torch.cuda.current_device():
        return contextlib.nullcontext()
    return torch.cuda.device(dev)


def _need_cuda(*ts):
    for t in ts:
        if t is not None and not t.is_cuda:
            raise ValueError("RAP kernels run on the GPU only: pass CUDA tensors (no CPU fallback)")


def _check(rc: int, what: str):
    if rc != 0:
        raise RapError(rc, what)


def _mask(sel, table) -> int:
    if isinstance(sel, int):
        return sel
    m = 0
    for x in sel:
        m |= 1 << (table[x] if isinstance(x, str) else int(x))
    return m


def perm_gen(seed: int, index: int = 0, w: int = 32) -> list[int]:
    """P = perm(seed, index, w) computed by the library on the host (rap_perm_gen): the P every
    transpose launch uses (index 0)."""
    buf = (ctypes.c_uint32 * w)()
    _check(lib().rap_perm_gen(seed, index, w, buf), "rap_perm_gen")
    return list(buf)


def perm_gen_batch(seed: int, count: int, w: int = 32, first_index: int = 0,
                   device="cuda", out: torch.Tensor | None = None) -> torch.Tensor:
    """Permutations P_n = perm(seed, n, w), n = first_index .. +count-1 -> uint8 [count, w], on the GPU."""
    if out is None:
        out = torch.empty((count, w), dtype=torch.uint8, device=device)
    _need_cuda(out)
    assert out.dtype == torch.uint8 and out.is_contiguous() and out.numel() == count * w
    with _on(out.device):
        _check(lib().rap_perm_gen_batch(seed, first_index, count, w, ctypes.c_void_p(out.data_ptr()),
                                        _stream(out)), "rap_perm_gen_batch")
    return out


def transpose(x: torch.Tensor, layout: str = "rap", seed: int = 0,
              out: torch.Tensor | None = None) -> torch.Tensor:
    """out[c, r] = x[r, c] (bit copy) via 32x32 shared-memory tiles in `layout`.

    x: 2-D CUDA tensor with 4- or 8-byte elements and unit inner stride.  out (optional):
    [cols, rows] tensor of the same dtype, unit inner stride, not overlapping x.
    """
    _need_cuda(x, out)
    if x.dim() != 2:
        raise ValueError("transpose expects a 2-D tensor")
    eb = x.element_size()
    if eb not in (4, 8):
        raise ValueError("transpose supports 4- and 8-byte elements")
    rows, cols = x.shape
    if x.stride(1) != 1 and rows * cols > 0:
        x = x.contiguous()
    if out is None:
        out = torch.empty((cols, rows), dtype=x.dtype, device=x.device)
    if out.shape != (cols, rows) or out.dtype != x.dtype or (out.stride(1) != 1 and rows * cols):
        raise ValueError("out must be a [cols, rows] tensor of x's dtype with unit inner stride")
    ld_src = x.stride(0) if rows > 1 else max(cols, 1)
    ld_dst = out.stride(0) if cols > 1 else max(rows, 1)
    with _on(x.device):
        _check(lib().rap_transpose(ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(out.data_ptr()),
                                   rows, cols, ld_src, ld_dst, eb, LAYOUTS[layout], seed,
                                   _stream(x)), "rap_transpose")
    return out


def transpose_host(x: torch.Tensor, out: torch.Tensor | None = None, layout: str = "rap", seed: int = 0,
                   workspace_bytes: int = 128 << 20, device="cuda") -> torch.Tensor:
    """End-to-end transpose of a HOST (ideally pinned) 2-D tensor into a host tensor [cols, rows]:
    row bands stream through the GPU with upload, RAP transpose and download overlapped.
    Synchronous.  A device workspace of `workspace_bytes` is taken from torch's allocator."""
    if x.is_cuda:
        raise ValueError("transpose_host takes host tensors; use transpose() for device tensors")
    if x.dim() != 2 or x.element_size() not in (4, 8) or x.stride(1) != 1:
        raise ValueError("transpose_host expects a 2-D host tensor of 4/8-byte elements, unit inner stride")
    rows, cols = x.shape
    if out is None:
        out = torch.empty((cols, rows), dtype=x.dtype, pin_memory=x.is_pinned())
    if out.is_cuda or out.shape != (cols, rows) or out.dtype != x.dtype or (out.stride(1) != 1 and rows * cols):
        raise ValueError("out must be a host [cols, rows] tensor of x's dtype with unit inner stride")
    dev = torch.device(device) if not isinstance(device, torch.device) else device
    if dev.index is None:
        dev = torch.device("cuda", torch.cuda.current_device())
    eb = x.element_size()
    need = 4 * 32 * cols * eb
    ws = torch.empty(max(workspace_bytes, need), dtype=torch.uint8, device=dev)
    with _on(dev):
        _check(lib().rap_transpose_host(ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(out.data_ptr()), rows, cols,
                                        x.stride(0) if rows > 1 else cols, out.stride(0) if cols > 1 else rows, eb,
                                        LAYOUTS[layout], seed, ctypes.c_void_p(ws.data_ptr()), ws.numel(),
                                        _stream(ws)), "rap_transpose_host")
    return out


def transpose_to_peers(shard: torch.Tensor, peer_ptrs, rank: int, ld_dst: int | None = None,
                       layout: str = "rap", seed: int = 0) -> None:
    """Fused sharded transpose (NEXT-2): this rank's row block [M, N] straight into every rank's
    output shard.  peer_ptrs: G device addresses (ints) of the [M, ld_dst] output shards, valid in
    this process.  Enqueue only -- the caller barriers across ranks before reading its shard."""
    _need_cuda(shard)
    M, N = shard.shape
    G = len(peer_ptrs)
    if shard.stride(1) != 1:
        raise ValueError("shard needs unit inner stride")
    arr = (ctypes.c_void_p * G)(*[ctypes.c_void_p(int(p)) for p in peer_ptrs])
    with _on(shard.device):
        _check(lib().rap_transpose_to_peers(ctypes.c_void_p(shard.data_ptr()), M, N, shard.stride(0) if M > 1 else N,
                                            arr, G, rank, N if ld_dst is None else ld_dst, shard.element_size(),
                                            LAYOUTS[layout], seed, _stream(shard)), "rap_transpose_to_peers")


def congestion(rows: torch.Tensor, cols: torch.Tensor, scheme: str = "rap",
               shift: torch.Tensor | None = None, w: int | None = None,
               out: torch.Tensor | None = None) -> torch.Tensor:
    """DMM congestion of n warps: rows/cols/shift int32 or uint32 CUDA [n, w] -> uint32 [n]."""
    _need_cuda(rows, cols, shift, out)
    n, ww = rows.shape
    w = ww if w is None else w
    assert ww == w and cols.shape == rows.shape
    for t in (rows, cols) + ((shift,) if shift is not None else ()):
        assert t.dtype in (torch.int32, torch.uint32) and t.is_contiguous()
    if shift is not None:
        assert shift.shape == rows.shape
    if out is None:
        out = torch.empty(n, dtype=torch.uint32, device=rows.device)
    with _on(rows.device):
        _check(lib().rap_congestion(w, n, ctypes.c_void_p(rows.data_ptr()),
                                    ctypes.c_void_p(cols.data_ptr()), SCHEMES[scheme],
                                    ctypes.c_void_p(shift.data_ptr() if shift is not None else 0),
                                    ctypes.c_void_p(out.data_ptr()), _stream(rows)),
               "rap_congestion")
    return out


def congestion_sweep(n_trials: int, seed: int, w: int = 32, patterns=("contiguous", "stride",
                     "diagonal", "random", "malicious"), schemes=("raw", "ras", "rap"),
                     first_trial: int = 0, out: torch.Tensor | None = None,
                     device="cuda", algo: str = "default") -> torch.Tensor:
    """Monte-Carlo congestion histogram int64 [npat, nsch, w+1], ACCUMULATED into `out`.

    algo: "default" (bit-sliced lane-mode Fisher-Yates + ballot histogram) or "match"
    (warp shuffle Fisher-Yates + __match_any_sync, the measured ablation); identical results.
    """
    pm, sm = _mask(patterns, PATTERNS), _mask(schemes, SCHEMES)
    shape = (bin(pm).count("1"), bin(sm).count("1"), w + 1)
    if out is None:
        out = torch.zeros(shape, dtype=torch.int64, device=device)
    _need_cuda(out)
    assert tuple(out.shape) == shape and out.dtype == torch.int64 and out.is_contiguous()
    with _on(out.device):
        _check(lib().rap_congestion_sweep_algo(w, pm, sm, seed, first_trial, n_trials,
                                               ctypes.c_void_p(out.data_ptr()), SWEEP_ALGOS[algo],
                                               _stream(out)), "rap_congestion_sweep")
    return out


def congestion_trace(cells: torch.Tensor, n_trials: int, seed: int, schemes=("raw", "ras", "rap"),
                     first_trial: int = 0, out: torch.Tensor | None = None) -> torch.Tensor:
    """cells int32/uint32 CUDA [n_warps, w] (row*w+col) -> int64 [nsch, w+1] (accumulated)."""
    _need_cuda(cells, out)
    n, w = cells.shape
    assert cells.dtype in (torch.int32, torch.uint32) and cells.is_contiguous()
    sm = _mask(schemes, SCHEMES)
    shape = (bin(sm).count("1"), w + 1)
    if out is None:
        out = torch.zeros(shape, dtype=torch.int64, device=cells.device)
    assert tuple(out.shape) == shape and out.dtype == torch.int64 and out.is_contiguous()
    with _on(cells.device):
        _check(lib().rap_congestion_trace(w, n, ctypes.c_void_p(cells.data_ptr()), sm, seed,
                                          first_trial, n_trials, ctypes.c_void_p(out.data_ptr()),
                                          _stream(cells)), "rap_congestion_trace")
    return out


def unpack_blocks(recv: torch.Tensor, out: torch.Tensor, G: int) -> torch.Tensor:
    """After the all-to-all of the sharded transpose: out[x, s*M + a] = recv[s*M + x, a].

    recv: CUDA [G*M, M] (source-ordered M x M blocks); out: CUDA [M, >= G*M] with unit inner stride.
    """
    _need_cuda(recv, out)
    GM, M = recv.shape
    assert GM == G * M and recv.is_contiguous() and out.dtype == recv.dtype
    assert out.shape[0] == M and out.shape[1] >= G * M and out.stride(1) == 1
    eb = recv.element_size()
    with _on(recv.device):
        _check(lib().rap_unpack_blocks(ctypes.c_void_p(recv.data_ptr()), ctypes.c_void_p(out.data_ptr()),
                                       G, M, out.stride(0) if M > 1 else G * M, eb, _stream(recv)),
               "rap_unpack_blocks")
    return out


def smem_transpose_bench(algorithm: str, scheme: str, elem_bytes: int = 4, seed: int = 0,
                         n_blocks: int = 1, reps: int = 1, device="cuda"):
    """Table III on this GPU: (logical result uint32 [n_blocks, 32, 32], cycles int64 [n_blocks])."""
    out = torch.empty((n_blocks, 32, 32), dtype=torch.int32, device=device)
    cyc = torch.empty(n_blocks, dtype=torch.int64, device=device)
    with _on(out.device):
        _check(lib().rap_smem_transpose_bench(SMEM_ALGORITHMS[algorithm], SCHEMES[scheme], elem_bytes, seed,
                                              n_blocks, reps, ctypes.c_void_p(out.data_ptr()),
                                              ctypes.c_void_p(cyc.data_ptr()), _stream(out)),
               "rap_smem_transpose_bench")
    return out, cyc


def congestion_sweep4(n_trials: int, seed: int, w: int = 32, patterns=tuple(PATTERNS4), schemes=tuple(SCHEMES4),
                      first_trial: int = 0, out: torch.Tensor | None = None, device="cuda") -> torch.Tensor:
    """§VII sweep over a w^4 array (Table IV): int64 [npat, nsch, w+1], ACCUMULATED into `out`."""
    pm, sm = _mask(patterns, PATTERNS4), _mask(schemes, SCHEMES4)
    shape = (bin(pm).count("1"), bin(sm).count("1"), w + 1)
    if out is None:
        out = torch.zeros(shape, dtype=torch.int64, device=device)
    _need_cuda(out)
    assert tuple(out.shape) == shape and out.dtype == torch.int64 and out.is_contiguous()
    with _on(out.device):
        _check(lib().rap_congestion_sweep4(w, pm, sm, seed, first_trial, n_trials, ctypes.c_void_p(out.data_ptr()),
                                           _stream(out)), "rap_congestion_sweep4")
    return out


def smem_gather_bench(src_index: torch.Tensor, layout: str = "rap", seed: int = 0, n_blocks: int = 1, reps: int = 1):
    """NEXT-4: apply a 32x32-tile gather `reps` times in shared memory under `layout`.
    src_index: CUDA int16/uint16 [1024].  Returns (final array int32 [n_blocks, 1024], cycles [n_blocks])."""
    _need_cuda(src_index)
    assert src_index.numel() == 1024 and src_index.element_size() == 2 and src_index.is_contiguous()
    out = torch.empty((n_blocks, 1024), dtype=torch.int32, device=src_index.device)
    cyc = torch.empty(n_blocks, dtype=torch.int64, device=src_index.device)
    with _on(out.device):
        _check(lib().rap_smem_gather_bench(ctypes.c_void_p(src_index.data_ptr()), LAYOUTS[layout], seed, n_blocks,
                                           reps, ctypes.c_void_p(out.data_ptr()), ctypes.c_void_p(cyc.data_ptr()),
                                           _stream(out)), "rap_smem_gather_bench")
    return out, cyc
