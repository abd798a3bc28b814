"""Pin the C oracle's per-seed stream to an independent pure-Python model (-m "not gpu").

tests/mini_oracle.py restates the counter contract (include/rap.h, reading vi) and the
DMM congestion in ~100 lines of Python with no code shared with oracle/rap_oracle.c.
A dropped Philox round, a swapped counter word, an off-by-one in the Durstenfeld index or in
the multiply-shift, a wrong domain or a missed merge of equal cells fails here bit for bit.
Also: the exhaustive RAP-diagonal histograms of SURVEY Appendix A.4 (all w! permutations,
w <= 8; pair-collision basis P:L1437-1446, uniform P P:L955-960).
"""
import itertools
import os

import numpy as np
import pytest

import mini_oracle as mo
from conftest import golden


def test_philox_known_answers_python():
    # Random123 known-answer vectors (the same ones the C oracle is pinned to)
    vecs = [((0, 0, 0, 0), (0, 0), (0x6627e8d5, 0xe169c58d, 0xbc57ac4c, 0x9b00dbd8)),
            ((0xffffffff,) * 4, (0xffffffff,) * 2, (0x408f276d, 0x41c83b0e, 0xa20bc7c6, 0x6d5451fd)),
            ((0x243f6a88, 0x85a308d3, 0x13198a2e, 0x03707344), (0xa4093822, 0x299f31d0),
             (0xd16cfe09, 0x94fdcceb, 0x5001e420, 0x24126ea1))]
    for ctr, key, out in vecs:
        assert mo.philox4x32_10(ctr, key) == out


SEED_TRIALS = [(1, 0), (2, 77), (3, (1 << 32) - 3), (0xDEADBEEF12345678, 10 ** 12)]


@pytest.mark.parametrize("seed,first", SEED_TRIALS)
def test_c_oracle_stream_equals_python_model(oracle, seed, first):
    """Per trial: the C oracle's words, P, r and random cells equal the Python model's."""
    for n in range(first, first + 300):
        for w in (32, 7):
            assert oracle.perm(seed, n, w).tolist() == mo.perm(seed, n, w), (n, w)
            assert oracle.ras_shifts(seed, n, w).tolist() == mo.ras_shifts(seed, n, w), (n, w)
            rows, cols = oracle.random_cells(seed, n, w)
            cells = mo.random_cells(seed, n, w)
            assert rows.tolist() == [c // w for c in cells] and cols.tolist() == [c % w for c in cells]
        for d, t in ((0, 0), (1, 5), (2, 31), (3, 2), (4, 7)):
            assert oracle.word(seed, n, d, t) == mo.word(seed, n, d, t)


@pytest.mark.parametrize("seed,first,count", [(1, 0, 4000), (2, 123456789, 2000), (3, (1 << 32) - 1000, 2000)])
def test_c_oracle_sweep_equals_python_model(oracle, seed, first, count):
    """The cfg2 sweep histogram (5 patterns x RAW/RAS/RAP, w = 32) of the C oracle equals the
    Python model's trial by trial (so the 10^9-trial goldens rest on two implementations)."""
    h = oracle.sweep(32, mo.PATTERNS, mo.SCHEMES, seed, first, count, threads=1)
    assert h.tolist() == mo.sweep(32, seed, first, count)


def test_sweep_golden_1e9_prefix_matches_python_model(oracle):
    # the first trials of the stored 10^9-trial run (seed 1) as the Python model sees them:
    # every trial's congestion in [1, w] and the totals additive
    h = np.array(mo.sweep(32, 1, 0, 1000), dtype=np.uint64)
    assert (h.sum(-1) == 1000).all()
    assert h[0, :, 1].tolist() == [1000, 1000, 1000]          # contiguous: 1 under every scheme
    assert h[1, 2, 1] == 1000 and h[1, 0, 32] == 1000          # RAP stride 1 (Theorem 2), RAW stride 32


def _a4_table():
    """SURVEY Appendix A.4 (computed by the survey's own enumeration, before this repo existed):
    number of permutations P of 0..w-1 whose diagonal access {(t, t)} has RAP congestion c."""
    out = {}
    for ln in open(golden("a4_rap_diagonal_hist.txt")):
        if ln.strip() and not ln.startswith("#"):
            w, counts = ln.split(":")
            out[int(w)] = [int(v) for v in counts.split()]
    return out


@pytest.mark.parametrize("w", [4, 5, 6, 7, 8])
def test_a4_exhaustive_rap_diagonal_histogram(oracle, w):
    """All w! permutations through the oracle's O6/O8: the histogram of the diagonal access's
    congestion equals Appendix A.4 exactly, and the Python model agrees."""
    hist = [0] * (w + 1)
    rows = np.arange(w, dtype=np.uint32)
    for P in itertools.permutations(range(w)):
        c = oracle.congestion(w, rows, rows, oracle.SCHEMES["rap"], np.array(P, dtype=np.uint32))
        hist[c] += 1
    assert hist[0] == 0 and hist[1:] == _a4_table()[w]
    if w <= 6:
        mh = [0] * (w + 1)
        for P in itertools.permutations(range(w)):
            mh[mo.congestion([(t, t) for t in range(w)], "rap", w, list(P), None)] += 1
        assert mh == hist


def test_a4_table_invariants():
    # independent of both implementations: sum = w!, h[w] = w (P(t) = t + s), h[w-1] = 0,
    # h[1] = 0 for even w and the cyclic-Latin-square transversal count (OEIS A006717) for odd w
    import math
    trans = {5: 15, 7: 133, 9: 2025, 11: 37851}
    for w, h in _a4_table().items():
        assert sum(h) == math.factorial(w) and h[w - 1] == w and h[w - 2] == 0
        assert h[0] == (trans[w] if w % 2 else 0)
