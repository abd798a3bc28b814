"""Pins of the §VII (higher-dimensional RAP, Table IV) part of the oracle.

Table IV is garbled in the extraction; what survives and is checked here: every scheme has
congestion 1 for contiguous access; RAW is w for the three stride accesses; 1P is 1 for Stride1
and w for Stride2 / Stride3; R1P and 3P are 1 for all three strides (for EVERY permutation);
the paper's R1P example -- the 6 permutations of (x, y, z) hit one bank -- holds for every P;
RAS strides and random access follow the balls-into-bins closed forms.
"""
import itertools
import math

import numpy as np
import pytest

from closed_forms import (balls_in_bins_cdf, expectation, pmf_from_cdf, random_access_cdf_cells,
                          variance)

S = {"raw": 0, "ras": 1, "1p": 2, "r1p": 3, "3p": 4}
PAT = {"contiguous": 0, "stride1": 1, "stride2": 2, "stride3": 3, "random": 4, "malicious": 5}


def test_address4_layout(oracle):
    # a[i][j][k][l] at address i w^3 + j w^2 + k w + l, in bank l
    w = 5
    for i, j, k, l in itertools.product(range(w), repeat=4):
        a = oracle.address4(S["raw"], w, i, j, k, l)
        assert a == ((i * w + j) * w + k) * w + l and a % w == l


def test_shift_functions(oracle):
    # 1P f = P[k]; R1P f = P[i]+P[j]+P[k]; 3P f = P[i]+Q[j]+R[k] (mod w)
    w = 7
    P, Q, R = np.random.default_rng(0).permuted(np.tile(np.arange(w), (3, 1)), axis=1)
    for i, j, k in itertools.product(range(w), repeat=3):
        base = ((i * w + j) * w + k) * w
        assert oracle.address4(S["1p"], w, i, j, k, 0, P, Q, R) == base + P[k] % w
        assert oracle.address4(S["r1p"], w, i, j, k, 0, P, Q, R) == base + (P[i] + P[j] + P[k]) % w
        assert oracle.address4(S["3p"], w, i, j, k, 0, P, Q, R) == base + (P[i] + Q[j] + R[k]) % w


@pytest.mark.parametrize("w", [4, 5, 6])
def test_table4_deterministic_entries_for_every_permutation(oracle, w):
    rng = np.random.default_rng(w)
    expect = {  # (pattern, scheme) -> congestion that must hold for every P (Table IV)
        ("contiguous", "raw"): 1, ("contiguous", "1p"): 1, ("contiguous", "r1p"): 1, ("contiguous", "3p"): 1,
        ("stride1", "raw"): w, ("stride2", "raw"): w, ("stride3", "raw"): w,
        ("stride1", "1p"): 1, ("stride2", "1p"): w, ("stride3", "1p"): w,
        ("stride1", "r1p"): 1, ("stride2", "r1p"): 1, ("stride3", "r1p"): 1,
        ("stride1", "3p"): 1, ("stride2", "3p"): 1, ("stride3", "3p"): 1,
    }
    for P in itertools.permutations(range(w)):
        Q, R = rng.permutation(w), rng.permutation(w)
        for (pat, sch), c in expect.items():
            cells = oracle.pattern4(PAT[pat], S[sch], w)
            assert oracle.congestion4(w, cells, S[sch], P, Q, R) == c, (pat, sch, P)


def test_r1p_six_permutation_groups(oracle):
    # a[x][y][z][l] and its 5 index permutations all go to bank
    # (P[x] + P[y] + P[z] + l) mod w under R1P -- for every P.  With one group (w = 6..8) the
    # malicious access therefore has congestion exactly 6.
    for w in (6, 7, 8):
        rng = np.random.default_rng(w)
        for _ in range(300):
            P = rng.permutation(w)
            cells = oracle.pattern4(PAT["malicious"], S["r1p"], w)
            banks = {oracle.address4(S["r1p"], w, *c, P=P) % w for c in cells[:6]}
            assert banks == {(P[0] + P[1] + P[2]) % w}
            assert oracle.congestion4(w, cells, S["r1p"], P) == 6


def _E(h):
    h = np.asarray(h, dtype=np.float64)
    c = np.arange(h.shape[-1])
    n = h.sum(-1)
    mu = (h * c).sum(-1) / n
    return mu, n


def test_sweep4_ras_and_random_closed_forms(oracle):
    w, N = 16, 60000
    h = oracle.sweep4(w, ["stride1", "stride3", "random"], ["ras", "3p"], 5, 0, N)
    pmf = pmf_from_cdf(balls_in_bins_cdf, w)
    E, sd = float(expectation(pmf)), float(variance(pmf)) ** 0.5
    for pi in (0, 1):                                   # RAS strides: w independent uniform banks
        mu, n = _E(h[pi, 0])
        assert abs(mu - E) < 2.576 * sd / math.sqrt(n)
    pr = pmf_from_cdf(lambda ww, m: random_access_cdf_cells(ww, m, ww ** 3), w)
    Er, sdr = float(expectation(pr)), float(variance(pr)) ** 0.5
    for si in (0, 1):                                   # random access: any scheme
        mu, n = _E(h[2, si])
        assert abs(mu - Er) < 2.576 * sdr / math.sqrt(n)
    # 3P strides are exactly 1 on every trial
    assert h[0, 1, 1] == N and h[1, 1, 1] == N


def test_random_cells_closed_form_matches_2d_special_case():
    # cells_per_bank = w reduces to the 2-D closed form (an identity of the two formulas)
    from closed_forms import random_access_cdf
    for w in (2, 3, 5):
        for m in range(w + 1):
            assert random_access_cdf_cells(w, m, w) == random_access_cdf(w, m)
