"""Closed forms the oracle is pinned against -- independent mathematics, not the oracle.

* ``balls_in_bins_cdf``: RAS stride / diagonal access.  With independent uniform shifts
  r_0..r_{w-1} the w requests of a stride access, one per row, land in
  independent uniform banks: w balls into w bins.  Pr[max load <= m] =
  w!/w^w [x^w] (sum_{k<=m} x^k/k!)^w  (exponential generating functions).
* ``random_access_cdf``: w cells drawn i.i.d. uniformly WITH replacement from the w^2 cells,
  equal addresses merged.  Each bank holds w cells, so
  Pr[max distinct-per-bank <= m] = w!/(w^2)^w [x^w] (sum_{k<=m} C(w,k) (e^x-1)^k)^w.
* transversal counts of the cyclic Latin square (OEIS A006717): the number of P with
  (t + P[t]) mod w all distinct, i.e. RAP diagonal congestion exactly 1.
"""
from fractions import Fraction
from math import comb, factorial


def _mul(a, b, n):
    out = [Fraction(0)] * (n + 1)
    for i, x in enumerate(a):
        if x == 0:
            continue
        for j, y in enumerate(b[: n + 1 - i]):
            if y:
                out[i + j] += x * y
    return out


def _pow(a, e, n):
    res = [Fraction(1)] + [Fraction(0)] * n
    base = a[:]
    while e:
        if e & 1:
            res = _mul(res, base, n)
        base = _mul(base, base, n)
        e >>= 1
    return res


def balls_in_bins_cdf(w: int, m: int) -> Fraction:
    egf = [Fraction(1, factorial(k)) if k <= m else Fraction(0) for k in range(w + 1)]
    return _pow(egf, w, w)[w] * factorial(w) / Fraction(w) ** w


def _exp_minus_one_pow(k: int, n: int):
    e1 = [Fraction(0)] + [Fraction(1, factorial(i)) for i in range(1, n + 1)]
    return _pow(e1, k, n)


def random_access_cdf(w: int, m: int) -> Fraction:
    n = w
    egf = [Fraction(0)] * (n + 1)
    for k in range(0, m + 1):
        term = _exp_minus_one_pow(k, n)
        c = comb(w, k)
        for i in range(n + 1):
            egf[i] += c * term[i]
    return _pow(egf, w, n)[n] * factorial(w) / Fraction(w * w) ** w


def pmf_from_cdf(cdf, w: int):
    """[Pr[C = c] for c = 0..w] from a cdf(w, m) function."""
    vals = [cdf(w, m) for m in range(w + 1)]
    return [vals[0]] + [vals[c] - vals[c - 1] for c in range(1, w + 1)]


def expectation(pmf):
    return sum(c * p for c, p in enumerate(pmf))


def variance(pmf):
    mu = expectation(pmf)
    return sum((c - mu) ** 2 * p for c, p in enumerate(pmf))


# OEIS A006717: transversals in the cyclic Latin square of order 2n+1 (n = 0..5).
CYCLIC_TRANSVERSALS_ODD = {1: 1, 3: 3, 5: 15, 7: 133, 9: 2025, 11: 37851}


def random_access_cdf_cells(w: int, m: int, cells_per_bank: int) -> Fraction:
    """w requests i.i.d. uniform over w * cells_per_bank cells (w banks of cells_per_bank cells
    each), equal cells merged: Pr[max distinct per bank <= m]
    = w!/(w*c)^w [x^w] (sum_{k<=m} C(c,k) (e^x-1)^k)^w."""
    n = w
    egf = [Fraction(0)] * (n + 1)
    for k in range(0, min(m, cells_per_bank) + 1):
        term = _exp_minus_one_pow(k, n)
        cc = comb(cells_per_bank, k)
        for i in range(n + 1):
            egf[i] += cc * term[i]
    return _pow(egf, w, n)[n] * factorial(w) / Fraction(w * cells_per_bank) ** w
