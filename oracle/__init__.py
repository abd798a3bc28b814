"""CPU oracle for the RAP hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product package
(``paper_conf_icppw_nakanomi14_b200``) never imports it, and this package imports
nothing from the product.  The arithmetic lives in ``rap_oracle.c`` (plain C, one
function per paper step, citations in its header); this module is ctypes marshalling.

Parity status:
  * philox / word ............ pinned (Random123 known-answer vectors)
  * perm ..................... pinned (permutation invariant, chi^2 uniformity, exhaustive E)
  * ras_shifts / random_cells  pinned (balls-into-bins closed forms, chi^2 of the sweep)
  * congestion / address ..... pinned (Fig.2, Fig.3, Thm 2, closed forms, brute force)
  * sweep .................... pinned (Tab.II within 99% CI, closed-form E, invariants)
  * transpose ................ pinned (Fig.5, numpy .T, involution)
  * rap_layout ............... pinned (Fig.6)
  * dmm_time ................. pinned (Fig.3, Lemma 1)
  * the exact per-seed stream (which Philox word feeds which draw) is a contract this
    repo defines (paper silent, reading vi): "parity unpinned" beyond that contract.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "rap_oracle.c")
_LIB = os.path.join(_HERE, "librap_oracle.so")

RAW, RAS, RAP, PAD, XOR = range(5)
SCHEMES = {"raw": RAW, "ras": RAS, "rap": RAP, "pad": PAD, "xor": XOR}
CONTIGUOUS, STRIDE, DIAGONAL, RANDOM, MALICIOUS = range(5)
PATTERNS = {"contiguous": CONTIGUOUS, "stride": STRIDE, "diagonal": DIAGONAL,
            "random": RANDOM, "malicious": MALICIOUS}
D_FY, D_RAS, D_RANDOM = 0, 1, 2


def build(force: bool = False) -> str:
    """Compile rap_oracle.c with gcc (-O2 -fopenmp).  Building the checker is not using it."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c99", "-fopenmp", "-fPIC", "-shared",
                               "-Wall", "-Wextra", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build())
        u32, u64, i64, p = ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int64, ctypes.c_void_p
        L.oracle_philox4x32_10.argtypes = [p, p, p]
        L.oracle_philox4x32_10.restype = None
        L.oracle_word.argtypes = [u64, u64, u32, u32]
        L.oracle_word.restype = u32
        L.oracle_perm.argtypes = [u64, u64, u32, p]
        L.oracle_ras_shifts.argtypes = [u64, u64, u32, p]
        L.oracle_random_cells.argtypes = [u64, u64, u32, p, p]
        L.oracle_address.argtypes = [u32, u32, u32, u32, p]
        L.oracle_address.restype = i64
        L.oracle_congestion.argtypes = [u32, u32, p, p, u32, p, p]
        L.oracle_pattern_cells.argtypes = [u32, u32, u32, u64, u64, p, p]
        L.oracle_sweep.argtypes = [u32, u32, u32, u64, u64, u64, p, ctypes.c_int]
        L.oracle_transpose.argtypes = [p, p, i64, i64, i64, i64, u32, ctypes.c_int]
        L.oracle_rap_layout.argtypes = [u32, p, p, p]
        L.oracle_dmm_time.argtypes = [p, u32, u32]
        L.oracle_dmm_time.restype = i64
        L.oracle_max_threads.argtypes = []
        L.oracle_perm_domain.argtypes = [u64, u64, u32, u32, p]
        L.oracle_shift4.argtypes = [u32, u32, u32, u32, u32, p, p, p, u64, u64]
        L.oracle_shift4.restype = i64
        L.oracle_address4.argtypes = [u32, u32, u32, u32, u32, u32, p, p, p, u64, u64]
        L.oracle_address4.restype = i64
        L.oracle_congestion4.argtypes = [u32, u32, p, p, p, p, u32, p, p, p, u64, u64, p]
        L.oracle_pattern4.argtypes = [u32, u32, u32, u64, u64, p, p, p, p]
        L.oracle_sweep4.argtypes = [u32, u32, u32, u64, u64, u64, p, ctypes.c_int]
        L.oracle_gather_power.argtypes = [p, u32, u32, p]
        for name in ("oracle_perm", "oracle_ras_shifts", "oracle_random_cells", "oracle_congestion",
                     "oracle_pattern_cells", "oracle_sweep", "oracle_transpose", "oracle_rap_layout",
                     "oracle_max_threads", "oracle_perm_domain", "oracle_congestion4", "oracle_pattern4",
                     "oracle_sweep4", "oracle_gather_power"):
            getattr(L, name).restype = ctypes.c_int
        _lib = L
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _check(rc: int, what: str):
    if rc != 0:
        raise ValueError(f"oracle {what} rejected its arguments (rc={rc})")


def max_threads() -> int:
    return int(lib().oracle_max_threads())


def philox4x32_10(ctr, key) -> np.ndarray:
    c = np.ascontiguousarray(ctr, dtype=np.uint32)
    k = np.ascontiguousarray(key, dtype=np.uint32)
    out = np.zeros(4, dtype=np.uint32)
    lib().oracle_philox4x32_10(_ptr(c), _ptr(k), _ptr(out))
    return out


def word(seed: int, n: int, d: int, t: int) -> int:
    return int(lib().oracle_word(seed, n, d, t))


def perm(seed: int, n: int, w: int) -> np.ndarray:
    a = np.zeros(w, dtype=np.uint32)
    _check(lib().oracle_perm(seed, n, w, _ptr(a)), "perm")
    return a


def ras_shifts(seed: int, n: int, w: int) -> np.ndarray:
    r = np.zeros(w, dtype=np.uint32)
    _check(lib().oracle_ras_shifts(seed, n, w, _ptr(r)), "ras_shifts")
    return r


def random_cells(seed: int, n: int, w: int):
    rows = np.zeros(w, dtype=np.uint32)
    cols = np.zeros(w, dtype=np.uint32)
    _check(lib().oracle_random_cells(seed, n, w, _ptr(rows), _ptr(cols)), "random_cells")
    return rows, cols


def address(scheme: int, w: int, i: int, j: int, shift=None) -> int:
    s = None if shift is None else np.ascontiguousarray(shift, dtype=np.uint32)
    a = int(lib().oracle_address(scheme, w, i, j, None if s is None else _ptr(s)))
    if a < 0:
        raise ValueError("oracle address rejected its arguments")
    return a


def congestion(w: int, rows, cols, scheme: int, shift=None) -> int:
    r = np.ascontiguousarray(rows, dtype=np.uint32)
    c = np.ascontiguousarray(cols, dtype=np.uint32)
    assert r.shape == c.shape and r.ndim == 1
    s = None if shift is None else np.ascontiguousarray(shift, dtype=np.uint32)
    out = np.zeros(1, dtype=np.uint32)
    _check(lib().oracle_congestion(w, r.size, _ptr(r), _ptr(c), scheme,
                                   None if s is None else _ptr(s), _ptr(out)), "congestion")
    return int(out[0])


def pattern_cells(pattern: int, scheme: int, w: int, seed: int = 0, n: int = 0):
    rows = np.zeros(w, dtype=np.uint32)
    cols = np.zeros(w, dtype=np.uint32)
    _check(lib().oracle_pattern_cells(pattern, scheme, w, seed, n, _ptr(rows), _ptr(cols)),
           "pattern_cells")
    return rows, cols


def _mask(sel, table) -> int:
    m = 0
    for x in sel:
        m |= 1 << (table[x] if isinstance(x, str) else int(x))
    return m


def sweep(w: int, patterns, schemes, seed: int, first: int, n_trials: int,
          threads: int | None = None) -> np.ndarray:
    """Histogram u64[len(patterns)][len(schemes)][w+1] (patterns/schemes in enum order)."""
    pm, sm = _mask(patterns, PATTERNS), _mask(schemes, SCHEMES)
    npat, nsch = bin(pm).count("1"), bin(sm).count("1")
    hist = np.zeros((npat, nsch, w + 1), dtype=np.uint64)
    th = max_threads() if threads is None else threads
    _check(lib().oracle_sweep(w, pm, sm, seed, first, n_trials, _ptr(hist), th), "sweep")
    return hist


def transpose(src: np.ndarray, threads: int = 1, out: np.ndarray | None = None) -> np.ndarray:
    """Plain definition: dst[c][r] = src[r][c] on the raw bits of a 2-D array.  `out`: an optional
    preallocated contiguous [cols, rows] array of src's dtype (the timing harness reuses one, so
    that a measurement is not dominated by first-touch page faults of a fresh result array)."""
    assert src.ndim == 2
    s = src
    if s.strides[1] != s.itemsize or s.strides[0] % s.itemsize:
        s = np.ascontiguousarray(s)
    rows, cols = s.shape
    ld_src = s.strides[0] // s.itemsize if rows else cols
    if out is not None:
        assert out.shape == (cols, rows) and out.dtype == s.dtype and out.flags.c_contiguous
        dst = out
    else:
        dst = np.empty((cols, rows), dtype=s.dtype)
    _check(lib().oracle_transpose(_ptr(s), _ptr(dst), rows, cols, max(ld_src, cols),
                                  max(rows, 0), s.itemsize, threads), "transpose")
    return dst


def rap_layout(P, logical: np.ndarray) -> np.ndarray:
    P = np.ascontiguousarray(P, dtype=np.uint32)
    w = P.size
    lg = np.ascontiguousarray(logical, dtype=np.uint32).reshape(w, w)
    phys = np.zeros((w, w), dtype=np.uint32)
    _check(lib().oracle_rap_layout(w, _ptr(P), _ptr(lg), _ptr(phys)), "rap_layout")
    return phys


def dmm_time(congestions, latency: int) -> int:
    c = np.ascontiguousarray(congestions, dtype=np.uint32)
    t = int(lib().oracle_dmm_time(_ptr(c), c.size, latency))
    if t < 0:
        raise ValueError("oracle dmm_time rejected its arguments")
    return t


# ---------------------------------------------------------------- O13: w^4 arrays (paper §VII)
S4 = {"raw": 0, "ras": 1, "1p": 2, "r1p": 3, "3p": 4}
P4 = {"contiguous": 0, "stride1": 1, "stride2": 2, "stride3": 3, "random": 4, "malicious": 5}


def perm_domain(seed: int, n: int, w: int, d: int) -> np.ndarray:
    a = np.zeros(w, dtype=np.uint32)
    _check(lib().oracle_perm_domain(seed, n, w, d, _ptr(a)), "perm_domain")
    return a


def _u32(x, w):
    return np.ascontiguousarray(np.zeros(w, np.uint32) if x is None else x, dtype=np.uint32)


def address4(scheme: int, w: int, i, j, k, l, P=None, Q=None, R=None, seed=0, n=0) -> int:
    P, Q, R = _u32(P, w), _u32(Q, w), _u32(R, w)
    a = int(lib().oracle_address4(scheme, w, i, j, k, l, _ptr(P), _ptr(Q), _ptr(R), seed, n))
    if a < 0:
        raise ValueError("oracle address4 rejected its arguments")
    return a


def congestion4(w: int, cells, scheme: int, P=None, Q=None, R=None, seed=0, n=0) -> int:
    c = np.ascontiguousarray(cells, dtype=np.uint32).reshape(-1, 4)
    ci, cj, ck, cl = (np.ascontiguousarray(c[:, m]) for m in range(4))
    P, Q, R = _u32(P, w), _u32(Q, w), _u32(R, w)
    out = np.zeros(1, dtype=np.uint32)
    _check(lib().oracle_congestion4(w, c.shape[0], _ptr(ci), _ptr(cj), _ptr(ck), _ptr(cl), scheme, _ptr(P),
                                    _ptr(Q), _ptr(R), seed, n, _ptr(out)), "congestion4")
    return int(out[0])


def pattern4(pattern: int, scheme: int, w: int, seed: int = 0, n: int = 0) -> np.ndarray:
    c = [np.zeros(w, dtype=np.uint32) for _ in range(4)]
    _check(lib().oracle_pattern4(pattern, scheme, w, seed, n, *[_ptr(x) for x in c]), "pattern4")
    return np.stack(c, 1)


def sweep4(w: int, patterns, schemes, seed: int, first: int, n_trials: int, threads: int | None = None):
    pm, sm = _mask(patterns, P4), _mask(schemes, S4)
    hist = np.zeros((bin(pm).count("1"), bin(sm).count("1"), w + 1), dtype=np.uint64)
    th = max_threads() if threads is None else threads
    _check(lib().oracle_sweep4(w, pm, sm, seed, first, n_trials, _ptr(hist), th), "sweep4")
    return hist


def gather_power(idx, reps: int) -> np.ndarray:
    """x_{k+1}[o] = x_k[idx[o]] applied `reps` times to x_0[o] = o (NEXT-4 reference)."""
    i = np.ascontiguousarray(idx, dtype=np.uint16)
    out = np.zeros(i.size, dtype=np.uint32)
    _check(lib().oracle_gather_power(_ptr(i), i.size, reps, _ptr(out)), "gather_power")
    return out
