"""Seeded synthetic inputs shared by the tests, smoke() and bench.py.

This module holds none of the method's arithmetic (no RNG contract of the sweep, no bank
maps, no transpose): it only fabricates input tensors and names the BASELINE.json configs.
Both the CUDA path and the oracle consume what it returns; neither is imported here.

Input recipe:
  * transpose matrices: uniformly random 32/64-bit patterns (torch.Generator, seeded), so
    NaNs with payloads, +-Inf, -0 and subnormals all occur; the first elements are forced to
    those special values so every run contains them.  The transpose is a bit copy, so the
    value distribution only matters for proving that no float path touches the data.
  * trace cells: per-warp access traces of the paper's pattern families (P:L592-603,
    L765-772) plus uniform random cells.
"""
from __future__ import annotations

import numpy as np
import torch

# BASELINE.json configs (index = position in BASELINE.json "configs")
CONFIGS = {
    0: dict(name="cfg1_tile32_f32_rap", kind="transpose", rows=32, cols=32, dtype="float32", layout="rap"),
    1: dict(name="cfg2_sweep_w32", kind="sweep", w=32, n_trials=10 ** 9),
    2: dict(name="cfg3_8192_f32", kind="transpose", rows=8192, cols=8192, dtype="float32", layout="rap"),
    3: dict(name="cfg4_16384_f64", kind="transpose", rows=16384, cols=16384, dtype="float64", layout="rap"),
    4: dict(name="cfg5_32768_f32_sharded", kind="dist_transpose", rows=32768, cols=32768, dtype="float32",
            layout="rap"),
}

_SPECIAL32 = [0x7FC00001, 0xFFC12345, 0x7F800000, 0xFF800000, 0x80000000, 0x00000000,
              0x00000001, 0x807FFFFF, 0x7F7FFFFF, 0x3F800000]
_SPECIAL64 = [0x7FF8000000000001, 0xFFF0000000000ABC, 0x7FF0000000000000, 0xFFF0000000000000,
              0x8000000000000000, 0x0, 0x1, 0x800FFFFFFFFFFFFF, 0x7FEFFFFFFFFFFFFF,
              0x3FF0000000000000]


def _bits_dtype(dtype: torch.dtype) -> torch.dtype:
    return {torch.float32: torch.int32, torch.int32: torch.int32, torch.uint32: torch.int32,
            torch.float64: torch.int64, torch.int64: torch.int64, torch.uint64: torch.int64}[dtype]


def random_bits(rows: int, cols: int, dtype=torch.float32, seed: int = 0, device="cpu",
                ld: int | None = None) -> torch.Tensor:
    """[rows, cols] tensor of `dtype` whose raw bits are uniform; optional row pitch `ld`."""
    ld = cols if ld is None else ld
    bd = _bits_dtype(dtype)
    gen = torch.Generator(device=device).manual_seed(seed)
    nbits = 32 if bd == torch.int32 else 64
    lo, hi = -(2 ** (nbits - 1)), 2 ** (nbits - 1) - 1
    buf = torch.randint(lo, hi, (rows * ld if rows else 0,), generator=gen, dtype=bd, device=device)
    special = _SPECIAL32 if bd == torch.int32 else _SPECIAL64
    k = min(len(special), buf.numel())
    if k:
        sv = [(v - (1 << nbits)) if v >= (1 << (nbits - 1)) else v for v in special[:k]]
        buf[:k] = torch.tensor(sv, dtype=bd, device=device)
    full = buf.view(dtype) if dtype != bd else buf
    return full.view(rows, ld)[:, :cols] if rows else full.view(0, cols)


def as_bits_numpy(t: torch.Tensor) -> np.ndarray:
    """Host numpy view of a tensor's raw bits (uint32/uint64), for bit-exact comparisons."""
    t = t.detach().cpu()
    bd = {4: torch.int32, 8: torch.int64}[t.element_size()]
    a = t.contiguous().view(bd).numpy()
    return a.view(np.uint32 if t.element_size() == 4 else np.uint64)


def trace_cells(n_warps: int, w: int = 32, seed: int = 0, device="cpu") -> torch.Tensor:
    """[n_warps, w] int32 cells row*w+col: a mix of row, column, diagonal, anti-diagonal,
    permutation-matrix and uniform-random warps (the paper's pattern families)."""
    rng = np.random.default_rng(seed)
    t = np.arange(w)
    out = np.empty((n_warps, w), dtype=np.int64)
    for k in range(n_warps):
        kind = k % 6
        a = int(rng.integers(w))
        if kind == 0:
            r, c = np.full(w, a), t
        elif kind == 1:
            r, c = t, np.full(w, a)
        elif kind == 2:
            r, c = t, (t + a) % w
        elif kind == 3:
            r, c = t, (a - t) % w
        elif kind == 4:
            r, c = t, rng.permutation(w)
        else:
            cells = rng.integers(0, w * w, size=w)
            r, c = cells // w, cells % w
        out[k] = r * w + c
    return torch.from_numpy(out.astype(np.int32)).to(device)


def tile_gather_patterns(seed: int = 0):
    """NEXT-4 inputs: 1024-entry source-index tables of a 32 x 32 tile (thread o = 32 s + t of
    warp s reads element src[o]).  Each table is a permutation of the tile; the adversarial ones
    put all 32 reads of a warp into one bank of a deterministic layout (finding 9):
      identity   warp s reads row s                      (contiguous)
      transpose  warp s reads column s                   (stride; RAW's worst case)
      diagonal   warp s reads (t, (t + s) mod 32)        (RAP's worst case, ~3.61)
      antidiag   warp s reads (t, (s - t) mod 32)        (+1 padding: (row + col) constant -> 32-way)
      xordiag    warp s reads (t, t xor s)               (XOR swizzle: col xor row constant -> 32-way)
      random     a seeded uniformly random permutation
    """
    t = np.arange(32)
    tabs = {}
    rows = lambda f: np.concatenate([f(s) for s in range(32)]).astype(np.uint16)
    tabs["identity"] = np.arange(1024, dtype=np.uint16)
    tabs["transpose"] = rows(lambda s: t * 32 + s)
    tabs["diagonal"] = rows(lambda s: t * 32 + (t + s) % 32)
    tabs["antidiag"] = rows(lambda s: t * 32 + (s - t) % 32)
    tabs["xordiag"] = rows(lambda s: t * 32 + (t ^ s))
    tabs["random"] = np.random.default_rng(seed).permutation(1024).astype(np.uint16)
    return tabs
