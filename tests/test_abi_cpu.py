"""Host-side checks of the C ABI that need no GPU (-m "not gpu").

librap.so must load, export every function include/rap.h declares, validate arguments
BEFORE touching CUDA, and -- with no GPU present -- fail with RAP_ERR_CUDA instead of
computing anything on the CPU (there is no CPU fallback).
"""
import ctypes
import os
import re

import pytest
import torch

from conftest import ROOT

import paper_conf_icppw_nakanomi14_b200 as rap
from paper_conf_icppw_nakanomi14_b200 import build as rbuild

OK, INVALID, UNSUPPORTED, ALIAS, CUDA = 0, 1, 2, 3, 4


@pytest.fixture(scope="module")
def L():
    rbuild.build()
    return rap.lib()


def header_functions():
    src = open(os.path.join(ROOT, "include", "rap.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(rap_[a-z_]+)\s*\(", src)))


def test_exports_every_declared_symbol(L):
    names = header_functions()
    assert {"rap_perm_gen", "rap_transpose", "rap_congestion", "rap_congestion_sweep",
            "rap_congestion_trace", "rap_status_str", "rap_abi_version"} <= set(names)
    for n in names:
        assert hasattr(L, n), n
    assert L.rap_abi_version() == 2


def test_status_strings(L):
    for s in range(5):
        assert L.rap_status_str(s).decode().startswith("RAP_")


P = ctypes.c_void_p


def test_transpose_validation(L):
    a, b = P(0x10000000), P(0x20000000)
    s = P(0)
    assert L.rap_transpose(a, b, 4, 4, 4, 4, 3, 4, 0, s) == INVALID      # elem_bytes
    assert L.rap_transpose(a, b, 4, 4, 4, 4, 4, 9, 0, s) == INVALID      # layout
    assert L.rap_transpose(a, b, 4, 4, 4, 4, 4, 7, 0, s) == INVALID      # layout
    assert L.rap_transpose(a, b, 4, 4, 4, 4, 4, 6, 0, s) == UNSUPPORTED  # RAP64 needs 8-byte elements
    assert L.rap_transpose(a, b, 4, 4, 4, 4, 4, 5, 0, s) == UNSUPPORTED  # RAP16 needs 8-byte elements
    assert L.rap_transpose(a, b, -1, 4, 4, 4, 4, 4, 0, s) == INVALID     # rows < 0
    assert L.rap_transpose(a, b, 4, 8, 4, 4, 4, 4, 0, s) == INVALID      # ld_src < cols
    assert L.rap_transpose(a, b, 8, 4, 4, 4, 4, 4, 0, s) == INVALID      # ld_dst < rows
    assert L.rap_transpose(P(0), b, 4, 4, 4, 4, 4, 4, 0, s) == INVALID   # null
    assert L.rap_transpose(P(0x10000002), b, 4, 4, 4, 4, 4, 4, 0, s) == INVALID  # misaligned
    assert L.rap_transpose(a, P(0x10000020), 4, 4, 4, 4, 4, 4, 0, s) == ALIAS
    assert L.rap_transpose(a, b, 0, 4, 4, 4, 4, 4, 0, s) == OK          # empty: no-op
    assert L.rap_transpose(a, b, 1 << 62, 1 << 62, 1 << 62, 1 << 62, 8, 4, 0, s) == INVALID


@pytest.mark.skipif(torch.cuda.is_available(), reason="checks the no-GPU behaviour")
def test_valid_calls_fail_loudly_without_gpu(L):
    # a well-formed request reaches CUDA and fails there: nothing is computed on the host
    a, b = P(0x10000000), P(0x20000000)
    assert L.rap_transpose(a, b, 64, 64, 64, 64, 4, 4, 0, P(0)) == CUDA
    assert L.rap_congestion_sweep(32, 31, 7, 1, 0, 1000, P(0x30000000), P(0)) == CUDA
    assert L.rap_perm_gen_batch(1, 0, 10, 32, P(0x30000000), P(0)) == CUDA


def test_sweep_validation(L):
    h, s = P(0x30000000), P(0)
    assert L.rap_congestion_sweep(1, 31, 7, 1, 0, 10, h, s) == INVALID    # w < 2
    assert L.rap_congestion_sweep(257, 31, 7, 1, 0, 10, h, s) == INVALID  # w > 256
    assert L.rap_congestion_sweep(32, 0, 7, 1, 0, 10, h, s) == INVALID    # empty pattern mask
    assert L.rap_congestion_sweep(32, 32, 7, 1, 0, 10, h, s) == INVALID   # unknown pattern
    assert L.rap_congestion_sweep(32, 31, 64, 1, 0, 10, h, s) == INVALID  # unknown scheme
    assert L.rap_congestion_sweep(24, 31, 16, 1, 0, 10, h, s) == INVALID  # XOR needs 2^k
    assert L.rap_congestion_sweep(32, 31, 7, 1, 0, 10, P(0), s) == INVALID
    assert L.rap_congestion_sweep(32, 31, 7, 1, 0, 0, P(0), s) == OK      # no trials: no-op
    L.rap_congestion_sweep_algo.argtypes = [ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32,
                                            ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64,
                                            ctypes.c_void_p, ctypes.c_uint32, ctypes.c_void_p]
    assert L.rap_congestion_sweep_algo(32, 31, 7, 1, 0, 10, h, 2, s) == INVALID   # unknown algo
    assert L.rap_congestion_sweep_algo(32, 31, 7, 1, 0, 0, h, 1, s) == OK
    assert L.rap_congestion_sweep_algo(64, 31, 7, 1, 0, 10, h, 1, s) == UNSUPPORTED  # match kernel: w <= 32


def test_congestion_trace_perm_validation(L):
    d, s = P(0x30000000), P(0)
    assert L.rap_congestion(1, 4, d, d, 2, d, d, s) == INVALID
    assert L.rap_congestion(32, 4, d, d, 7, d, d, s) == INVALID
    assert L.rap_congestion(32, 4, d, d, 2, P(0), d, s) == INVALID        # RAP needs shifts
    assert L.rap_congestion(12, 4, d, d, 4, None, d, s) == INVALID        # XOR needs 2^k
    assert L.rap_congestion(32, 0, d, d, 2, d, d, s) == OK
    assert L.rap_congestion_trace(32, 4, d, 0, 1, 0, 5, d, s) == INVALID
    assert L.rap_congestion_trace(32, 4, P(0), 7, 1, 0, 5, d, s) == INVALID
    assert L.rap_congestion_trace(32, 0, d, 7, 1, 0, 5, d, s) == OK
    assert L.rap_perm_gen_batch(1, 0, 4, 33, d, s) == INVALID
    assert L.rap_perm_gen_batch(1, 0, 4, 1, d, s) == INVALID
    assert L.rap_perm_gen_batch(1, 0, 4, 32, P(0), s) == INVALID
    assert L.rap_perm_gen_batch(1, 0, 0, 32, P(0), s) == OK
    buf = (ctypes.c_uint32 * 300)()
    assert L.rap_perm_gen(1, 0, 1, buf) == INVALID                       # w < 2
    assert L.rap_perm_gen(1, 0, 257, buf) == INVALID                     # w > 256
    assert L.rap_perm_gen(1, 0, 32, None) == INVALID


@pytest.mark.parametrize("w", [2, 3, 5, 16, 31, 32, 33, 64, 100, 256])
def test_host_perm_gen_matches_oracle(L, oracle, w):
    """§8(b) rap_perm_gen (host, the P every transpose launch passes to its kernel) equals the
    oracle's O3 Durstenfeld permutation for many (seed, index): a pure host call, no GPU."""
    import numpy as np
    for seed in (0, 1, 77, (1 << 64) - 1):
        for index in (0, 1, 2, 12345, (1 << 32) + 7, (1 << 64) - 1):
            assert np.array_equal(np.array(rap.perm_gen(seed, index, w)), oracle.perm(seed, index, w)), \
                (seed, index, w)


def test_smem_bench_and_unpack_validation(L):
    d, s = P(0x30000000), P(0)
    L.rap_smem_transpose_bench.argtypes = [ctypes.c_uint32, ctypes.c_int, ctypes.c_uint32, ctypes.c_uint64,
                                           ctypes.c_uint32, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_void_p,
                                           ctypes.c_void_p]
    assert L.rap_smem_transpose_bench(3, 2, 4, 0, 1, 1, d, d, s) == INVALID      # unknown algorithm
    assert L.rap_smem_transpose_bench(0, 3, 4, 0, 1, 1, d, d, s) == INVALID      # PAD not in Table III
    assert L.rap_smem_transpose_bench(0, 2, 2, 0, 1, 1, d, d, s) == INVALID      # elem_bytes
    assert L.rap_smem_transpose_bench(0, 2, 4, 0, 0, 1, P(0), P(0), s) == OK     # no blocks
    L.rap_unpack_blocks.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64, ctypes.c_int64,
                                    ctypes.c_int64, ctypes.c_uint32, ctypes.c_void_p]
    assert L.rap_unpack_blocks(d, P(0x40000000), 2, 8, 15, 4, s) == INVALID      # ld_out < G*M
    assert L.rap_unpack_blocks(d, P(0x30000010), 2, 8, 16, 4, s) == ALIAS
    assert L.rap_unpack_blocks(d, P(0x40000000), 2, 8, 16, 3, s) == INVALID
    assert L.rap_unpack_blocks(d, P(0x40000000), 0, 8, 16, 4, s) == OK


def test_transpose_to_peers_validation(L):
    f = L.rap_transpose_to_peers
    f.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.POINTER(ctypes.c_void_p),
                  ctypes.c_uint32, ctypes.c_uint32, ctypes.c_int64, ctypes.c_uint32, ctypes.c_int, ctypes.c_uint64,
                  ctypes.c_void_p]
    peers = (ctypes.c_void_p * 2)(0x40000000, 0x50000000)
    src, s = P(0x10000000), P(0)
    assert f(src, 64, 128, 128, peers, 2, 2, 128, 4, 4, 0, s) == INVALID     # rank >= G
    assert f(src, 48, 96, 96, peers, 2, 0, 96, 4, 4, 0, s) == INVALID        # M not a multiple of 32
    assert f(src, 64, 100, 128, peers, 2, 0, 128, 4, 4, 0, s) == INVALID     # N != G*M
    assert f(src, 64, 128, 128, peers, 17, 0, 128, 4, 4, 0, s) == INVALID    # too many peers
    assert f(src, 64, 128, 128, peers, 2, 0, 100, 4, 4, 0, s) == INVALID     # ld_dst < N
    alias = (ctypes.c_void_p * 2)(0x10000000, 0x50000000)
    assert f(src, 64, 128, 128, alias, 2, 0, 128, 4, 4, 0, s) == ALIAS
    assert f(src, 64, 128, 128, peers, 2, 0, 128, 8, 5, 0, s) == UNSUPPORTED  # RAP16: local transpose only


def test_sweep4_validation(L):
    h, s = P(0x30000000), P(0)
    f = L.rap_congestion_sweep4
    f.argtypes = [ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_uint64,
                  ctypes.c_uint64, ctypes.c_void_p, ctypes.c_void_p]
    assert f(3, 63, 31, 1, 0, 10, h, s) == INVALID
    assert f(33, 63, 31, 1, 0, 10, h, s) == INVALID
    assert f(32, 64, 31, 1, 0, 10, h, s) == INVALID
    assert f(32, 63, 32, 1, 0, 10, h, s) == INVALID
    assert f(32, 63, 31, 1, 0, 0, P(0), s) == OK


def test_python_binding_refuses_cpu_tensors(L):
    x = torch.zeros(8, 8)
    with pytest.raises(ValueError):
        rap.transpose(x)
    with pytest.raises(ValueError):
        rap.congestion_sweep(10, 1, out=torch.zeros(5, 3, 33, dtype=torch.int64))


def test_product_does_not_import_oracle():
    # the product package and the oracle share no code and never import each other
    pkg = os.path.join(ROOT, "paper_conf_icppw_nakanomi14_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, f)).read()
                assert not re.search(r"\b(import|from)\s+oracle\b|librap_oracle|rap_oracle\.c|oracle_\w+\(", txt), f
    for f in os.listdir(os.path.join(ROOT, "oracle")):
        if f.endswith((".py", ".c")):
            txt = open(os.path.join(ROOT, "oracle", f)).read()
            assert "import paper_conf" not in txt and "csrc" not in txt and "rap.h" not in txt, f
