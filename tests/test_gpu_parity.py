"""GPU parity: the CUDA path (through the C ABI / binding) against the CPU oracle (-m gpu).

Integer and bit work, so every comparison is bit-exact: transposed bytes (as uint32/uint64
views, including NaN payloads, -0, Inf, subnormals), permutations, per-warp congestions and
per-seed u64 histograms.
"""
import itertools
import math
import os

import numpy as np
import pytest
import torch

import workloads
from closed_forms import balls_in_bins_cdf, expectation, pmf_from_cdf, random_access_cdf, variance

pytestmark = pytest.mark.gpu

LAYOUT_NAMES = ["raw", "pad", "xor", "ras", "rap"]
ALL_PAT = ["contiguous", "stride", "diagonal", "random", "malicious"]
ALL_SCH = ["raw", "ras", "rap", "pad", "xor"]


@pytest.fixture(scope="module")
def rap():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_icppw_nakanomi14_b200 as r
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    return r


def bits(t):
    return workloads.as_bits_numpy(t)


# ------------------------------------------------------------------ T0 permutations
@pytest.mark.parametrize("w", [2, 3, 5, 16, 31, 32])
def test_perm_gen_matches_oracle(rap, oracle, w):
    first, count = 12345678901, 3000
    P = rap.perm_gen_batch(seed=77, count=count, w=w, first_index=first).cpu().numpy()
    for k in range(count):
        assert np.array_equal(P[k], oracle.perm(77, first + k, w).astype(np.uint8)), k
    assert all(sorted(row) == list(range(w)) for row in P.tolist())


def test_perm_gen_batch_1e6_indices(rap, oracle):
    """10^6 consecutive indices (straddling 2^32, so the counter's high word changes) at w = 32,
    every permutation compared with the oracle's O3, and the host call (rap_perm_gen) agrees."""
    first, count = (1 << 32) - 500_000, 1_000_000
    P = rap.perm_gen_batch(seed=3, count=count, w=32, first_index=first).cpu().numpy()
    for k in range(count):
        assert np.array_equal(P[k], oracle.perm(3, first + k, 32)), k
    for k in range(0, count, 9973):
        assert rap.perm_gen(3, first + k, 32) == P[k].tolist()


# ------------------------------------------------------------------ T1-T3 transpose
SHAPES = [(1, 1), (1, 100), (100, 1), (32, 32), (33, 65), (64, 32), (257, 129), (1000, 3), (5, 1000),
          (96, 4096)]


@pytest.mark.parametrize("layout", LAYOUT_NAMES)
@pytest.mark.parametrize("dtype", [torch.float32, torch.float64])
def test_transpose_shapes(rap, oracle, layout, dtype):
    for i, (r, c) in enumerate(SHAPES):
        x = workloads.random_bits(r, c, dtype, seed=i)
        y = rap.transpose(x.cuda(), layout=layout, seed=i + 11)
        torch.cuda.synchronize()
        assert y.shape == (c, r)
        assert np.array_equal(bits(y), oracle.transpose(bits(x))), (layout, r, c)


@pytest.mark.parametrize("layout", ["rap", "raw", "xor"])
@pytest.mark.parametrize("dtype", [torch.float32, torch.float64])
def test_transpose_strided_and_misaligned(rap, oracle, layout, dtype):
    # row pitch ld_src > cols (vector path when 16B-aligned), an odd column offset (scalar
    # path), and an output with row pitch ld_dst > rows
    big = workloads.random_bits(300, 260, dtype, seed=3)
    for (r0, c0, r1, c1) in [(0, 0, 300, 256), (3, 4, 291, 250), (1, 1, 200, 77), (2, 3, 35, 40)]:
        xs = big.cuda()[r0:r1, c0:c1]
        out_big = torch.zeros((c1 - c0, (r1 - r0) + 9), dtype=dtype, device="cuda")
        out = out_big[:, 5:5 + (r1 - r0)]
        rap.transpose(xs, layout=layout, seed=1, out=out)
        torch.cuda.synchronize()
        assert np.array_equal(bits(out), oracle.transpose(bits(big[r0:r1, c0:c1])))
        assert not bits(out_big[:, :5]).any() and not bits(out_big[:, 5 + (r1 - r0):]).any()


def test_transpose_empty_and_alias(rap):
    x = torch.zeros((0, 7), device="cuda")
    assert rap.transpose(x).shape == (7, 0)
    buf = torch.zeros(64 * 64 * 2, device="cuda")
    with pytest.raises(rap.RapError):
        rap.transpose(buf[:4096].view(64, 64), out=buf[2048:2048 + 4096].view(64, 64))


def test_transpose_result_independent_of_seed(rap):
    x = workloads.random_bits(200, 300, torch.float32, seed=9).cuda()
    ref = rap.transpose(x, layout="raw")
    for s in (0, 1, 2, 2 ** 63 + 5):
        assert torch.equal(rap.transpose(x, layout="rap", seed=s).view(torch.int32), ref.view(torch.int32))


def _full_check(oracle, x_dev, y_dev):
    """Every element: the oracle transposes the whole matrix (multi-threaded plain loops)."""
    assert np.array_equal(bits(y_dev), oracle.transpose(bits(x_dev), threads=oracle.max_threads()))


def _band_check(oracle, x_dev, y_dev, n_bands=6, band=48, seed=0):
    """Full-size check on sampled row bands: the oracle transposes each band of x."""
    rows, cols = x_dev.shape
    rng = np.random.default_rng(seed)
    starts = sorted(set([0, rows - band] + rng.integers(0, rows - band, n_bands).tolist()))
    for r0 in starts:
        xb = bits(x_dev[r0:r0 + band])
        yb = bits(y_dev[:, r0:r0 + band])
        assert np.array_equal(yb, oracle.transpose(xb)), r0


@pytest.mark.parametrize("layout", LAYOUT_NAMES)
def test_transpose_cfg3_8192_f32(rap, oracle, layout):
    # BASELINE cfg3 at full size, in the launch configuration bench.py times
    x = workloads.random_bits(8192, 8192, torch.float32, seed=0, device="cuda")
    y = rap.transpose(x, layout=layout, seed=0)
    torch.cuda.synchronize()
    _full_check(oracle, x, y)
    # property at any size: transposing twice is the identity (bit-exact)
    z = rap.transpose(y, layout=layout, seed=1)
    assert torch.equal(z.view(torch.int32), x.view(torch.int32))


def test_transpose_beyond_2pow32_elements(rap, oracle):
    # 65600 x 65600 fp32 = 4.3e9 elements (17.2 GB each way): every element offset needs 64 bits;
    # ragged in both dimensions (65600 = 2050 tiles, not a multiple of the 16 x 2 cluster super-tile)
    n = 65600
    x = workloads.random_bits(n, n, torch.float32, seed=21, device="cuda")
    y = rap.transpose(x, layout="rap", seed=4)
    torch.cuda.synchronize()
    _band_check(oracle, x, y, n_bands=2, band=33, seed=3)
    for c0 in (0, 40000, n - 17):
        assert np.array_equal(bits(y[c0:c0 + 17]), oracle.transpose(bits(x[:, c0:c0 + 17]))), c0
    z = rap.transpose(y, layout="rap", seed=5)
    assert torch.equal(z.view(torch.int32), x.view(torch.int32))


@pytest.mark.parametrize("shape", [((1 << 27) + 5, 3), (3, (1 << 27) + 5), ((1 << 22) + 1, 33)])
def test_transpose_extreme_aspect(rap, oracle, shape):
    # tall / wide extremes: one partial tile column or row over millions of tiles
    x = workloads.random_bits(*shape, torch.float64, seed=22, device="cuda")
    y = rap.transpose(x, layout="rap", seed=6)
    torch.cuda.synchronize()
    assert np.array_equal(bits(y), oracle.transpose(bits(x), threads=oracle.max_threads()))


@pytest.mark.parametrize("layout", ["rap", "rap64", "rap16"])
def test_transpose_cfg4_16384_f64(rap, oracle, layout):
    # BASELINE cfg4 at full size, in the launch configuration bench.py times: all 2^28 doubles
    # compared with the oracle (rap64: the w = 32 map on 8-byte slots, the headline; rap: the
    # w = 32 map on two 32-bit planes; rap16: RAP over 16 double banks)
    x = workloads.random_bits(16384, 16384, torch.float64, seed=0, device="cuda")
    y = rap.transpose(x, layout=layout, seed=0)
    torch.cuda.synchronize()
    _full_check(oracle, x, y)
    z = rap.transpose(y, layout=layout, seed=9)
    assert torch.equal(z.view(torch.int64), x.view(torch.int64))


@pytest.mark.parametrize("layout", ["raw", "pad", "xor", "ras"])
def test_transpose_cfg4_16384_f64_baselines(rap, layout):
    # the baseline layouts (two 32-bit planes) at cfg4 size: equal to the RAP result (itself
    # checked in full against the oracle above) and an involution
    x = workloads.random_bits(16384, 16384, torch.float64, seed=0, device="cuda")
    ref = rap.transpose(x, layout="rap", seed=0)
    y = rap.transpose(x, layout=layout, seed=3)
    assert torch.equal(y.view(torch.int64), ref.view(torch.int64))


def test_transpose64_seeds_and_ragged(rap, oracle):
    # the 8-byte-slot kernel under many P (the P^-1 drain lanes depend on P) on ragged shapes
    # spanning several 12-warp super-tiles
    for i, (r, c) in enumerate([(385, 33), (31, 1025), (800, 417), (1024, 96)]):
        x = workloads.random_bits(r, c, torch.float64, seed=200 + i)
        for seed in (0, 1, 2, 3, 12345, 2 ** 64 - 1):
            y = rap.transpose(x.cuda(), layout="rap64", seed=seed)
            torch.cuda.synchronize()
            assert np.array_equal(bits(y), oracle.transpose(bits(x))), (r, c, seed)


def test_transpose_rap64_shapes(rap, oracle):
    for i, (r, c) in enumerate(SHAPES + [(384, 64), (385, 33)]):
        x = workloads.random_bits(r, c, torch.float64, seed=300 + i)
        y = rap.transpose(x.cuda(), layout="rap64", seed=i)
        torch.cuda.synchronize()
        assert np.array_equal(bits(y), oracle.transpose(bits(x))), (r, c)
    with pytest.raises(rap.RapError, match="UNSUPPORTED"):
        rap.transpose(torch.zeros((64, 64), device="cuda"), layout="rap64")


# T2b (ii): the RAP-16 double tile (8-byte elements only)
def test_transpose_rap16_shapes(rap, oracle):
    for i, (r, c) in enumerate(SHAPES + [(384, 64), (385, 33), (31, 1025)]):
        x = workloads.random_bits(r, c, torch.float64, seed=100 + i)
        y = rap.transpose(x.cuda(), layout="rap16", seed=i)
        torch.cuda.synchronize()
        assert np.array_equal(bits(y), oracle.transpose(bits(x))), (r, c)


def test_transpose_rap16_strided(rap, oracle):
    big = workloads.random_bits(300, 260, torch.float64, seed=4)
    for (r0, c0, r1, c1) in [(0, 0, 300, 256), (3, 1, 291, 250), (2, 3, 35, 40)]:
        xs = big.cuda()[r0:r1, c0:c1]
        out_big = torch.zeros((c1 - c0, (r1 - r0) + 9), dtype=torch.float64, device="cuda")
        out = out_big[:, 3:3 + (r1 - r0)]
        rap.transpose(xs, layout="rap16", seed=2, out=out)
        torch.cuda.synchronize()
        assert np.array_equal(bits(out), oracle.transpose(bits(big[r0:r1, c0:c1])))
        assert not bits(out_big[:, :3]).any() and not bits(out_big[:, 3 + (r1 - r0):]).any()


def test_transpose_rap16_rejects_32bit(rap):
    with pytest.raises(rap.RapError, match="UNSUPPORTED"):
        rap.transpose(torch.zeros((64, 64), device="cuda"), layout="rap16")


def test_transpose_cfg1_tile(rap, oracle):
    for seed in (0, 1, 2):
        x = workloads.random_bits(32, 32, torch.float32, seed=seed)
        y = rap.transpose(x.cuda(), layout="rap", seed=seed)
        torch.cuda.synchronize()
        assert np.array_equal(bits(y), oracle.transpose(bits(x)))


# ------------------------------------------------------------------ C3 batched evaluator
@pytest.mark.parametrize("w", [2, 4, 7, 16, 32])
def test_congestion_batched_matches_oracle(rap, oracle, w):
    rng = np.random.default_rng(w)
    n = 400
    rows = rng.integers(0, w, (n, w))
    cols = rng.integers(0, w, (n, w))
    # duplicates and structured warps
    rows[::5] = rows[::5, :1]
    cols[::7] = cols[::7, :1]
    rows[1::9], cols[1::9] = np.arange(w), np.arange(w)
    shift = np.stack([rng.permutation(w) for _ in range(n)])
    schemes = ["raw", "ras", "rap", "pad"] + (["xor"] if w & (w - 1) == 0 else [])
    t = lambda a: torch.from_numpy(a.astype(np.int32)).cuda()
    for s in schemes:
        got = rap.congestion(t(rows), t(cols), s, shift=t(shift)).cpu().numpy()
        for k in range(n):
            sh = shift[k] if s in ("ras", "rap") else None
            assert got[k] == oracle.congestion(w, rows[k], cols[k], oracle.SCHEMES[s], sh), (s, k)


def test_congestion_out_of_range_marks_zero(rap):
    rows = torch.zeros((2, 32), dtype=torch.int32, device="cuda")
    cols = torch.arange(32, dtype=torch.int32, device="cuda").repeat(2, 1)
    cols[1, 5] = 40
    got = rap.congestion(rows, cols, "raw").cpu().tolist()
    assert got == [1, 0]


# ------------------------------------------------------------------ C1-C4 sweep
@pytest.mark.parametrize("seed", [1, 2, 3])
def test_sweep_bit_exact_w32(rap, oracle, seed):
    N = 1_000_000
    g = rap.congestion_sweep(N, seed=seed, w=32, patterns=ALL_PAT, schemes=ALL_SCH)
    o = oracle.sweep(32, ALL_PAT, ALL_SCH, seed, 0, N)
    assert np.array_equal(g.cpu().numpy().astype(np.uint64), o)


@pytest.mark.parametrize("algo", ["default", "match"])
@pytest.mark.parametrize("w", [2, 3, 7, 16, 31, 32])
def test_sweep_bit_exact_other_w(rap, oracle, w, algo):
    N = 100_003
    sch = ["raw", "ras", "rap", "pad"] + (["xor"] if w & (w - 1) == 0 else [])
    g = rap.congestion_sweep(N, seed=5, w=w, patterns=ALL_PAT, schemes=sch, first_trial=2 ** 33 + 17,
                             algo=algo)
    o = oracle.sweep(w, ALL_PAT, sch, 5, 2 ** 33 + 17, N)
    assert np.array_equal(g.cpu().numpy().astype(np.uint64), o)


def test_sweep_algos_agree_tiny_ranges(rap, oracle):
    # ragged batches: n_trials not a multiple of 32, single trials, odd first_trial
    for first, n in ((0, 1), (5, 31), (31, 33), (1000, 65), (2 ** 40 + 3, 97)):
        a = rap.congestion_sweep(n, seed=12, first_trial=first, algo="default")
        b = rap.congestion_sweep(n, seed=12, first_trial=first, algo="match")
        o = oracle.sweep(32, ALL_PAT, ["raw", "ras", "rap"], 12, first, n)
        assert torch.equal(a, b)
        assert np.array_equal(a.cpu().numpy().astype(np.uint64), o)


def test_sweep_masks_and_chunks(rap, oracle):
    N = 200_000
    for pats, schs in ((["random"], ["rap"]), (["stride", "malicious"], ["ras", "xor"]),
                       (["diagonal"], ["raw", "pad"])):
        g = rap.congestion_sweep(N, seed=8, patterns=pats, schemes=schs, first_trial=99)
        o = oracle.sweep(32, pats, schs, 8, 99, N)
        assert np.array_equal(g.cpu().numpy().astype(np.uint64), o)
    # accumulation: arbitrary chunks sum to the one-shot histogram
    one = rap.congestion_sweep(N, seed=4)
    acc = torch.zeros_like(one)
    for a, b in ((0, 1), (1, 77777), (77777, 150001), (150001, N)):
        rap.congestion_sweep(b - a, seed=4, first_trial=a, out=acc)
    assert torch.equal(one, acc)


def test_sweep_full_size_1e9(rap, oracle):
    # BASELINE cfg2 at full size: 10^9 trials, w=32.  Properties that hold at any size plus
    # a sampled sub-range recomputed by the oracle.
    N = 10 ** 9
    h = rap.congestion_sweep(N, seed=1, patterns=ALL_PAT, schemes=["raw", "ras", "rap"]).cpu().numpy()
    assert (h.sum(-1) == N).all()
    assert h[0, :, 1].tolist() == [N, N, N]          # contiguous: 1 under every scheme
    assert h[1, 0, 32] == N and h[1, 2, 1] == N      # stride: RAW 32, RAP 1 (Theorem 2)
    assert h[2, 0, 1] == N                           # diagonal RAW 1
    assert np.array_equal(h[1, 1], h[4, 1]) and np.array_equal(h[2, 2], h[4, 2])
    c = np.arange(33)
    pmf = pmf_from_cdf(balls_in_bins_cdf, 32)
    E, sd = float(expectation(pmf)), float(variance(pmf)) ** 0.5
    mu = (h[1, 1] * c).sum() / N
    assert abs(mu - E) < 2.576 * sd / math.sqrt(N)   # ~3.53, 99% CI
    pmf_r = pmf_from_cdf(random_access_cdf, 32)
    Er, sdr = float(expectation(pmf_r)), float(variance(pmf_r)) ** 0.5
    for s in range(3):
        assert abs((h[3, s] * c).sum() / N - Er) < 2.576 * sdr / math.sqrt(N)
    mu_rap = (h[2, 2] * c).sum() / N
    assert round(mu_rap, 2) == 3.61                  # Table II RAP diagonal
    # sampled sub-range of the same run: bit-exact against the oracle
    first = 987_654_321
    g = rap.congestion_sweep(200_000, seed=1, first_trial=first)
    o = oracle.sweep(32, ALL_PAT, ["raw", "ras", "rap"], 1, first, 200_000)
    assert np.array_equal(g.cpu().numpy().astype(np.uint64), o)


def read_sweep_golden(path):
    """tests/golden/sweep_w32_1e9_seed<s>.txt (written by tools/oracle_golden_1e9.py from oracle/ only)."""
    import json
    meta, h = None, np.zeros((5, 3, 33), dtype=np.uint64)
    for ln in open(path):
        if ln.startswith("# {"):
            meta = json.loads(ln[2:])
        elif not ln.startswith("#") and ln.strip():
            f = ln.split()
            h[ALL_PAT.index(f[0]), ["raw", "ras", "rap"].index(f[1])] = [int(v) for v in f[2:]]
    return meta, h


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_sweep_1e9_bit_exact_per_seed(rap, seed):
    # BASELINE cfg2 at full size, the north star's "matches the oracle bit-for-bit per seed":
    # the whole 10^9-trial histogram of each seed against the oracle's (computed once on the
    # host cores by tools/oracle_golden_1e9.py, ~30 min per seed; stored under tests/golden)
    import conftest
    path = conftest.golden(f"sweep_w32_1e9_seed{seed}.txt")
    if not os.path.exists(path):
        pytest.skip(f"{path} not generated yet (python tools/oracle_golden_1e9.py)")
    meta, expect = read_sweep_golden(path)
    assert meta["n_trials"] == 10 ** 9 and meta["first_trial"] == 0 and meta["seed"] == seed
    g = rap.congestion_sweep(10 ** 9, seed=seed, patterns=ALL_PAT, schemes=["raw", "ras", "rap"])
    assert np.array_equal(g.cpu().numpy().astype(np.uint64), expect)
    # the same histogram assembled from 7 uneven launches (accumulation is exact)
    acc = torch.zeros_like(g)
    cuts = [0, 1, 31, 33, 10 ** 6 + 7, 123_456_789, 700_000_001, 10 ** 9]
    for a, b in zip(cuts[:-1], cuts[1:]):
        rap.congestion_sweep(b - a, seed=seed, first_trial=a, out=acc)
    assert torch.equal(acc, g)


# ------------------------------------------------------------------ trace evaluator
def test_trace_matches_oracle(rap, oracle):
    w, n_trials, first = 32, 40, 1000
    cells = workloads.trace_cells(30, w, seed=4)
    g = rap.congestion_trace(cells.cuda(), n_trials, seed=6, schemes=ALL_SCH, first_trial=first)
    expect = np.zeros((5, w + 1), dtype=np.uint64)
    cl = cells.numpy()
    for n in range(first, first + n_trials):
        P, r = oracle.perm(6, n, w), oracle.ras_shifts(6, n, w)
        for k in range(cl.shape[0]):
            rows, cols = cl[k] // w, cl[k] % w
            for si, s in enumerate(ALL_SCH):
                sh = {"ras": r, "rap": P}.get(s)
                expect[si, oracle.congestion(w, rows, cols, oracle.SCHEMES[s], sh)] += 1
    assert np.array_equal(g.cpu().numpy().astype(np.uint64), expect)


def _trace_oracle(oracle, cl, seed, first, n_trials, schemes, w=32):
    """Histogram of the oracle's direct DMM congestion (O8) per (trial, trace warp, scheme); a
    trace warp with a cell >= w*w counts in bin 0."""
    expect = np.zeros((len(schemes), w + 1), dtype=np.uint64)
    for n in range(first, first + n_trials):
        P, r = oracle.perm(seed, n, w), oracle.ras_shifts(seed, n, w)
        for k in range(cl.shape[0]):
            if (cl[k] >= w * w).any():
                expect[:, 0] += 1
                continue
            rows, cols = cl[k] // w, cl[k] % w
            for si, s in enumerate(schemes):
                expect[si, oracle.congestion(w, rows, cols, oracle.SCHEMES[s], {"ras": r, "rap": P}.get(s))] += 1
    return expect


@pytest.mark.parametrize("schemes", [["ras"], ["rap", "xor"], ["pad"], ["raw", "ras", "rap"], ALL_SCH])
def test_trace_w32_masks_ragged_invalid(rap, oracle, schemes):
    # ragged against the kernel's units (64 trace warps x 32 trials), a bad cell, every mask shape
    w, n_trials, first = 32, 70, 12345
    cells = workloads.trace_cells(131, w, seed=8)
    cells[77, 5] = w * w + 3
    g = rap.congestion_trace(cells.cuda(), n_trials, seed=9, schemes=schemes, first_trial=first)
    expect = _trace_oracle(oracle, cells.numpy(), 9, first, n_trials, schemes)
    assert np.array_equal(g.cpu().numpy().astype(np.uint64), expect)
    assert (g[:, 0] == n_trials).all()


def test_trace_bench_size_sampled_and_additive(rap, oracle):
    # the bench workload (4096 trace warps x 256 trials, five schemes): a 48-warp sample of it
    # against the oracle one by one, and additivity over trial ranges at full size
    cells = workloads.trace_cells(4096, 32, seed=0)
    rng = np.random.default_rng(5)
    pick = np.sort(rng.choice(4096, 48, replace=False))
    sub = cells[pick].contiguous()
    g = rap.congestion_trace(sub.cuda(), 256, seed=1, schemes=ALL_SCH)
    assert np.array_equal(g.cpu().numpy().astype(np.uint64), _trace_oracle(oracle, sub.numpy(), 1, 0, 256, ALL_SCH))
    cd = cells.cuda()
    full = rap.congestion_trace(cd, 256, seed=1, schemes=ALL_SCH)
    parts = rap.congestion_trace(cd, 100, seed=1, schemes=ALL_SCH)
    rap.congestion_trace(cd, 156, seed=1, schemes=ALL_SCH, first_trial=100, out=parts)
    assert torch.equal(full, parts) and (full.sum(-1) == 4096 * 256).all()


@pytest.mark.parametrize("w", [2, 5, 8, 16, 31])
def test_trace_small_w_matches_oracle(rap, oracle, w):
    # w < 32: lanes >= w idle, banks reduced mod w, w + 1 bins per scheme; ragged units, bad cell
    schemes = ["raw", "ras", "rap", "pad"] + (["xor"] if w & (w - 1) == 0 else [])
    cells = workloads.trace_cells(70, w, seed=w)
    cells[3, 0] = w * w                                  # invalid -> bin 0
    g = rap.congestion_trace(cells.cuda(), 45, seed=11, schemes=schemes, first_trial=77)
    expect = _trace_oracle(oracle, cells.numpy(), 11, 77, 45, schemes, w=w)
    assert np.array_equal(g.cpu().numpy().astype(np.uint64), expect)


def test_trace_small_w_and_invalid(rap, oracle):
    w = 8
    cells = workloads.trace_cells(13, w, seed=1)
    cells[3, 2] = w * w + 5                          # invalid -> bin 0
    g = rap.congestion_trace(cells.cuda(), 7, seed=2, schemes=["rap", "raw"]).cpu().numpy()
    assert g[:, 0].tolist() == [7, 7]
    assert (g.sum(-1) == 13 * 7).all()


# ------------------------------------------------------------------ T4 sharded transpose pieces
@pytest.mark.parametrize("dtype", [torch.float32, torch.float64])
@pytest.mark.parametrize("G,M", [(1, 64), (2, 96), (4, 64), (8, 33), (3, 50)])
def test_sharded_transpose_emulated_on_one_gpu(rap, oracle, dtype, G, M):
    # G virtual ranks on one device: local rap_transpose per shard, the all-to-all as block
    # slicing, rap_unpack_blocks per rank; the union must equal the oracle's A^T.
    N = G * M
    A = workloads.random_bits(N, N, dtype, seed=G * 100 + M)
    Ad = A.cuda()
    sends = [rap.transpose(Ad[g * M:(g + 1) * M].contiguous(), layout="rap", seed=3) for g in range(G)]
    outs = []
    for g in range(G):
        recv = torch.cat([sends[s][g * M:(g + 1) * M] for s in range(G)], 0).contiguous()
        outs.append(rap.unpack_blocks(recv, torch.empty((M, N), dtype=dtype, device="cuda"), G))
    got = torch.cat(outs, 0)
    torch.cuda.synchronize()
    assert np.array_equal(bits(got), oracle.transpose(bits(A)))


def _cfg5_check(oracle, A, got, seed):
    """32768^2 check of every element: the oracle transposes the whole 4 GiB matrix."""
    _full_check(oracle, A, got)


@pytest.mark.parametrize("G", [2, 4, 8])
def test_transpose_cfg5_32768_sharded_emulated(rap, oracle, G):
    # BASELINE cfg5 at full size (32768^2 float32, 4 GiB), the NCCL-path pieces of G ranks on one
    # GPU: per-rank local RAP transpose of its M x N row block, the all-to-all as block slicing,
    # rap_unpack_blocks into the rank's M x N output rows.
    N = 32768
    M = N // G
    A = workloads.random_bits(N, N, torch.float32, seed=50 + G, device="cuda")
    got = torch.empty((N, N), dtype=torch.float32, device="cuda")
    sends = [rap.transpose(A[s * M:(s + 1) * M], layout="rap", seed=3) for s in range(G)]   # N x M each
    for g in range(G):
        # rank g's receive buffer: block g (rows gM..gM+M) of every rank's send, in rank order
        recv = torch.cat([sends[s][g * M:(g + 1) * M] for s in range(G)], 0)
        rap.unpack_blocks(recv, got[g * M:(g + 1) * M], G)
        del recv
    del sends
    torch.cuda.synchronize()
    _cfg5_check(oracle, A, got, seed=G)
    # property at full size: the sharded result equals the 1-GPU transpose bit for bit
    assert torch.equal(got.view(torch.int32), rap.transpose(A, layout="raw").view(torch.int32))


def test_transpose_to_peers_cfg5_32768_emulated(rap, oracle):
    # NEXT-2 fused exchange at cfg5's full size, G = 8: every rank's kernel stores its tiles
    # straight into the owners' output shards (local buffers standing in for mapped peers)
    N, G = 32768, 8
    M = N // G
    A = workloads.random_bits(N, N, torch.float32, seed=77, device="cuda")
    got = torch.zeros((N, N), dtype=torch.float32, device="cuda")
    ptrs = [got[h * M:(h + 1) * M].data_ptr() for h in range(G)]
    for g in range(G):
        rap.transpose_to_peers(A[g * M:(g + 1) * M], ptrs, g, layout="rap", seed=5)
    torch.cuda.synchronize()
    _cfg5_check(oracle, A, got, seed=9)
    assert torch.equal(rap.transpose(got, layout="rap", seed=2).view(torch.int32), A.view(torch.int32))


def test_unpack_blocks_strided_output(rap):
    G, M = 3, 40
    recv = workloads.random_bits(G * M, M, torch.float32, seed=1).cuda()
    big = torch.zeros((M, G * M + 7), dtype=torch.float32, device="cuda")
    rap.unpack_blocks(recv, big, G)
    r = recv.view(torch.int32).view(G, M, M).cpu()
    b = big.view(torch.int32).cpu()
    for s in range(G):
        assert torch.equal(b[:, s * M:(s + 1) * M], r[s])
    assert not b[:, G * M:].any()


def test_dist_world1_nccl(rap, oracle):
    # the dist entry points under a real NCCL process group of size 1 (the 1-GPU box)
    import os
    import torch.distributed as dist
    from paper_conf_icppw_nakanomi14_b200 import dist as rdist
    os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
    os.environ.setdefault("MASTER_PORT", "29561")
    dist.init_process_group("nccl", rank=0, world_size=1)
    try:
        h = rdist.congestion_sweep(50_000, seed=2, first_trial=3)
        o = oracle.sweep(32, ALL_PAT, ["raw", "ras", "rap"], 2, 3, 50_000)
        assert np.array_equal(h.cpu().numpy().astype(np.uint64), o)
        A = workloads.random_bits(256, 256, torch.float32, seed=4)
        out = rdist.transpose_sharded(A.cuda())
        assert np.array_equal(bits(out), oracle.transpose(bits(A)))
    finally:
        dist.destroy_process_group()


# ------------------------------------------------------------------ NEXT-1 Table III kernels
@pytest.mark.parametrize("elem", [4, 8])
@pytest.mark.parametrize("alg", ["crsw", "srcw", "drdw"])
@pytest.mark.parametrize("scheme", ["raw", "ras", "rap"])
def test_smem_transpose_bench_results(rap, oracle, alg, scheme, elem):
    # each algorithm transposes; odd reps -> A^T, even reps -> A, for every CTA's P/r
    A = np.arange(1024, dtype=np.int32).reshape(32, 32)
    AT = oracle.transpose(A)
    o1, c1 = rap.smem_transpose_bench(alg, scheme, elem, seed=7, n_blocks=40, reps=5)
    o2, _ = rap.smem_transpose_bench(alg, scheme, elem, seed=7, n_blocks=40, reps=2)
    o1, o2 = o1.cpu().numpy(), o2.cpu().numpy()
    assert all(np.array_equal(o1[k], AT) for k in range(40))
    assert all(np.array_equal(o2[k], A) for k in range(40))
    assert (c1.cpu().numpy() > 0).all()


# ------------------------------------------------------------------ NEXT-2 fused exchange
@pytest.mark.parametrize("dtype", [torch.float32, torch.float64])
@pytest.mark.parametrize("G,M", [(1, 64), (2, 96), (4, 64), (8, 32), (3, 160)])
@pytest.mark.parametrize("layout", ["rap", "raw"])
def test_transpose_to_peers_emulated(rap, oracle, dtype, G, M, layout):
    # G virtual ranks on one GPU: "peer" output shards are local buffers; every rank's kernel
    # writes its tiles into the owners' shards.  The union must be the oracle's A^T.
    N = G * M
    A = workloads.random_bits(N, N, dtype, seed=G * 7 + M)
    Ad = A.cuda()
    outs = [torch.zeros((M, N), dtype=dtype, device="cuda") for _ in range(G)]
    ptrs = [o.data_ptr() for o in outs]
    for g in range(G):
        rap.transpose_to_peers(Ad[g * M:(g + 1) * M], ptrs, g, layout=layout, seed=5)
    torch.cuda.synchronize()
    assert np.array_equal(bits(torch.cat(outs, 0)), oracle.transpose(bits(A)))


def test_transpose_to_peers_padded_pitch(rap, oracle):
    G, M = 2, 64
    N = G * M
    A = workloads.random_bits(N, N, torch.float32, seed=3)
    outs = [torch.zeros((M, N + 8), dtype=torch.float32, device="cuda") for _ in range(G)]
    for g in range(G):
        rap.transpose_to_peers(A.cuda()[g * M:(g + 1) * M], [o.data_ptr() for o in outs], g, ld_dst=N + 8)
    torch.cuda.synchronize()
    got = torch.cat([o[:, :N] for o in outs], 0)
    assert np.array_equal(bits(got), oracle.transpose(bits(A)))
    assert not bits(torch.cat([o[:, N:] for o in outs], 0)).any()


def test_fused_transpose_symmetric_memory_world1(rap, oracle):
    # the host path of NEXT-2 (symmetric-memory rendezvous + barriers) under a real NCCL group
    import os
    import torch.distributed as dist
    from paper_conf_icppw_nakanomi14_b200 import dist as rdist
    os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
    os.environ.setdefault("MASTER_PORT", "29563")
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        A = workloads.random_bits(256, 256, torch.float32, seed=11)
        ft = rdist.FusedTranspose((256, 256), torch.float32)
        out = ft(A.cuda())
        torch.cuda.synchronize()
        assert np.array_equal(bits(out), oracle.transpose(bits(A)))
    finally:
        dist.destroy_process_group()


# ------------------------------------------------------------------ NEXT-3 wide DMM warps
@pytest.mark.parametrize("w", [33, 48, 64, 100, 128, 256])
def test_sweep_wide_bit_exact(rap, oracle, w):
    N = 3001 if w <= 128 else 1201
    sch = ["raw", "ras", "rap", "pad"] + (["xor"] if w & (w - 1) == 0 else [])
    g = rap.congestion_sweep(N, seed=21, w=w, patterns=ALL_PAT, schemes=sch, first_trial=2 ** 35 + 3)
    o = oracle.sweep(w, ALL_PAT, sch, 21, 2 ** 35 + 3, N)
    assert np.array_equal(g.cpu().numpy().astype(np.uint64), o)


@pytest.mark.parametrize("w", [16, 24, 64, 96, 256])
def test_sweep_default_masks_other_w(rap, oracle, w):
    # the compile-time-mask kernels (5 patterns x RAW/RAS/RAP) off w = 32: the w < 32 warp kernel
    # and the lane-mode wide kernel; trial count ragged against the 32-trial batches
    N = 2777 if w <= 96 else 997
    g = rap.congestion_sweep(N, seed=5, w=w, first_trial=12345)
    o = oracle.sweep(w, ALL_PAT, ["raw", "ras", "rap"], 5, 12345, N)
    assert np.array_equal(g.cpu().numpy().astype(np.uint64), o)


@pytest.mark.parametrize("w,N", [(64, 400_000), (128, 200_000), (256, 100_000)])
def test_table2_wide_columns_on_gpu(rap, w, N):
    # Table II columns w = 64, 128, 256 from the GPU sweep: every entry within
    # rounding (0.005) + the 99% Monte-Carlo interval; contiguous / RAP stride exactly 1.
    col = [16, 32, 64, 128, 256].index(w)
    import os
    from conftest import golden
    rows = [ln.split() for ln in open(golden("table2.txt")) if ln.strip() and not ln.startswith("#")]
    table = {(r[0], r[1]): float(r[2 + col]) for r in rows}
    pats, schs = ["contiguous", "stride", "diagonal", "random"], ["raw", "ras", "rap"]
    h = rap.congestion_sweep(N, seed=4, w=w, patterns=pats, schemes=schs).cpu().numpy().astype(np.float64)
    c = np.arange(w + 1)
    for pi, p in enumerate(pats):
        for si, s in enumerate(schs):
            mu = (h[pi, si] * c).sum() / N
            sd = np.sqrt((h[pi, si] * (c - mu) ** 2).sum() / N)
            assert abs(mu - table[(p, s)]) <= 0.005 + 2.576 * sd / math.sqrt(N) + 1e-12, (p, s, mu)
    assert h[0, :, 1].tolist() == [N] * 3 and h[1, 2, 1] == N


# ------------------------------------------------------------------ NEXT-3 §VII w^4 arrays
ALL_P4 = ["contiguous", "stride1", "stride2", "stride3", "random", "malicious"]
ALL_S4 = ["raw", "ras", "1p", "r1p", "3p"]


@pytest.mark.parametrize("w", [4, 6, 7, 16, 32])
def test_sweep4_bit_exact(rap, oracle, w):
    N = 20_000
    g = rap.congestion_sweep4(N, seed=8, w=w, first_trial=777)
    o = oracle.sweep4(w, ALL_P4, ALL_S4, 8, 777, N)
    assert np.array_equal(g.cpu().numpy().astype(np.uint64), o)


def test_sweep4_table4_entries_w32(rap):
    N = 1_000_000
    h = rap.congestion_sweep4(N, seed=3, w=32).cpu().numpy()
    one = lambda p, s: h[ALL_P4.index(p), ALL_S4.index(s), 1] == N
    full = lambda p, s: h[ALL_P4.index(p), ALL_S4.index(s), 32] == N
    for s in ALL_S4:
        assert one("contiguous", s)
    for p in ("stride1", "stride2", "stride3"):
        assert full(p, "raw") and one(p, "r1p") and one(p, "3p")
    assert one("stride1", "1p") and full("stride2", "1p") and full("stride3", "1p")
    # R1P malicious: every group of 6 hits one bank, so the congestion is a multiple of 6
    mal = h[ALL_P4.index("malicious"), ALL_S4.index("r1p")]
    assert mal.sum() == N and all(mal[c] == 0 for c in range(33) if c % 6)


# ------------------------------------------------------------------ NEXT-4 data-dependent gather
@pytest.mark.parametrize("layout", LAYOUT_NAMES)
def test_smem_gather_results(rap, oracle, layout):
    for name, idx in workloads.tile_gather_patterns(seed=3).items():
        for reps in (1, 3):
            out, cyc = rap.smem_gather_bench(torch.from_numpy(idx.view(np.int16)).cuda(), layout, seed=5,
                                             n_blocks=8, reps=reps)
            exp = oracle.gather_power(idx, reps)
            got = out.cpu().numpy().astype(np.uint32)
            assert all(np.array_equal(got[k], exp) for k in range(8)), (name, layout, reps)


# ------------------------------------------------------------------ host-to-host pipeline
@pytest.mark.parametrize("dtype", [torch.float32, torch.float64])
@pytest.mark.parametrize("shape,ws", [((1000, 300), 4 * 32 * 300 * 8), ((4096, 2048), 8 << 20),
                                      ((33, 65), 1 << 20), ((2048, 96), 3 * 32 * 96 * 8 * 4 + 1)])
def test_transpose_host_pipeline(rap, oracle, dtype, shape, ws):
    r, c = shape
    x = workloads.random_bits(r, c, dtype, seed=r + c).pin_memory()
    y = rap.transpose_host(x, layout="rap", seed=2, workspace_bytes=ws)
    assert np.array_equal(bits(y), oracle.transpose(bits(x)))


def test_transpose_host_strided_pageable(rap, oracle):
    big = workloads.random_bits(300, 260, torch.float32, seed=8)        # pageable, ld 260
    xs = big[:, :250]
    out_big = torch.zeros((250, 310), dtype=torch.float32)
    rap.transpose_host(xs, out=out_big[:, :300], workspace_bytes=1 << 20)
    assert np.array_equal(bits(out_big[:, :300]), oracle.transpose(bits(xs)))
    assert not bits(out_big[:, 300:]).any()


# ------------------------------------------------------------------ randomized shapes / pitches
def test_transpose_randomized_geometry(rap, oracle):
    # 60 seeded draws of (rows, cols, source pitch, source offset, destination pitch, dtype, layout):
    # vector and scalar load paths, partial super-tiles, padded output rows -- all bit-exact
    rng = np.random.default_rng(2024)
    for k in range(60):
        dtype = [torch.float32, torch.float64][k % 2]
        layout = LAYOUT_NAMES[k % 5]
        rows, cols = int(rng.integers(1, 700)), int(rng.integers(1, 700))
        pad_s, off = int(rng.integers(0, 9)), int(rng.integers(0, 5))
        pad_d = int(rng.integers(0, 9))
        big = workloads.random_bits(rows, cols + pad_s + off, dtype, seed=k).cuda()
        xs = big[:, off:off + cols]
        out_big = torch.zeros((cols, rows + pad_d), dtype=dtype, device="cuda")
        rap.transpose(xs, layout=layout, seed=k, out=out_big[:, :rows])
        torch.cuda.synchronize()
        assert np.array_equal(bits(out_big[:, :rows]), oracle.transpose(bits(xs))), (k, rows, cols, layout)
        if pad_d:
            assert not bits(out_big[:, rows:]).any()


# ------------------------------------------------------------------ programmatic dependent launch
@pytest.mark.parametrize("dtype,layout", [(torch.float32, "rap"), (torch.float64, "rap"), (torch.float64, "rap64"),
                                          (torch.float64, "rap16"), (torch.float32, "raw")])
def test_transpose_chains_under_pdl(rap, dtype, layout):
    """Back-to-back transposes on one stream, no host sync in between: a grid may load its source
    before its predecessor completes only when that source is not the predecessor's destination
    (pdl_early_loads).  Chains that read what the previous and the one-before-previous launches
    wrote, and a torch kernel rewriting a source in between, must all see finished data."""
    n = 4096
    bd = torch.int32 if dtype == torch.float32 else torch.int64
    xs = [workloads.random_bits(n, n, dtype, seed=40 + i, device="cuda") for i in range(6)]
    ys = [torch.empty_like(x) for x in xs]
    for _ in range(3):
        for x, y in zip(xs, ys):                       # independent launches: early loads
            rap.transpose(x, layout=layout, seed=1, out=y)
        z = rap.transpose(ys[3], layout=layout, seed=2)   # reads the output of 3 launches ago
        w = rap.transpose(z, layout=layout, seed=3)       # reads its predecessor's output
        u = rap.transpose(ys[5], layout=layout, seed=4)   # reads the output of 3 launches ago
        xs[0].view(bd).add_(1)                            # a torch kernel rewrites a source ...
        v = rap.transpose(xs[0], layout=layout, seed=5)   # ... that the next launch reads
        torch.cuda.synchronize()
        assert torch.equal(z.view(bd), xs[3].view(bd))
        assert torch.equal(w.view(bd), ys[3].view(bd))
        assert torch.equal(u.view(bd), xs[5].view(bd))
        assert torch.equal(v.view(bd), xs[0].t().contiguous().view(bd))
        for x, y in zip(xs[1:], ys[1:]):
            assert torch.equal(y.view(bd), x.t().contiguous().view(bd))
