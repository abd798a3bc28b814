"""A second, independent CPU model of the counter contract and the DMM congestion (test only).

Pure Python, written from the paper and the contract in include/rap.h / DESIGN.md reading vi,
sharing no code with oracle/rap_oracle.c: it exists to pin the C oracle's per-seed stream
(which permutation, which shifts, which random cells a trial draws) to something other than
itself.  Slow on purpose; used on <= 10^4 trials.

  word(seed, n, d, t) = Philox4x32-10(ctr = (n mod 2^32, n >> 32, t >> 2, d),
                                      key = (seed mod 2^32, seed >> 32))[t mod 4]
  P   = Durstenfeld shuffle of 0..w-1: for k = w-1 .. 1, j = floor(word(0, w-1-k) * (k+1) / 2^32),
        swap a[k], a[j]                          ("uniformly from all w! permutations")
  r_i = floor(word(1, i) * w / 2^32)             (RAS: independent random shifts)
  c_t = floor(word(2, t) * w^2 / 2^32)           (random access, with replacement; reading ii)
  bank of cell (i, j): RAW j, RAS (j + r_i) mod w, RAP (j + P_i) mod w
  congestion = max over banks of the number of DISTINCT cells requested in it
"""
M32 = 0xFFFFFFFF


def philox4x32_10(ctr, key):
    """Salmon et al. (SC'11) Philox4x32 with 10 rounds; multipliers / Weyl constants of Random123."""
    c0, c1, c2, c3 = ctr
    k0, k1 = key
    for rnd in range(10):
        if rnd:
            k0 = (k0 + 0x9E3779B9) & M32
            k1 = (k1 + 0xBB67AE85) & M32
        p0 = 0xD2511F53 * c0
        p1 = 0xCD9E8D57 * c2
        c0, c1, c2, c3 = ((p1 >> 32) ^ c1 ^ k0, p1 & M32, (p0 >> 32) ^ c3 ^ k1, p0 & M32)
    return (c0, c1, c2, c3)


def word(seed, n, d, t):
    blk = philox4x32_10((n & M32, n >> 32, t >> 2, d), (seed & M32, seed >> 32))
    return blk[t & 3]


def perm(seed, n, w):
    a = list(range(w))
    for k in range(w - 1, 0, -1):
        j = (word(seed, n, 0, w - 1 - k) * (k + 1)) >> 32
        a[k], a[j] = a[j], a[k]
    return a


def ras_shifts(seed, n, w):
    return [(word(seed, n, 1, i) * w) >> 32 for i in range(w)]


def random_cells(seed, n, w):
    return [(word(seed, n, 2, t) * w * w) >> 32 for t in range(w)]


def bank(scheme, w, i, j, P, r):
    if scheme == "raw":
        return j
    if scheme == "ras":
        return (j + r[i]) % w
    if scheme == "rap":
        return (j + P[i]) % w
    raise ValueError(scheme)


def congestion(cells, scheme, w, P, r):
    """cells: list of (row, col); duplicates merge (one request per distinct cell)."""
    per_bank = {}
    for (i, j) in set(cells):
        b = bank(scheme, w, i, j, P, r)
        per_bank[b] = per_bank.get(b, 0) + 1
    return max(per_bank.values())


def pattern(name, scheme, w, seed, n):
    if name == "contiguous":
        return [(0, t) for t in range(w)]
    if name == "stride":
        return [(t, 0) for t in range(w)]
    if name == "diagonal":
        return [(t, t) for t in range(w)]
    if name == "random":
        return [(c // w, c % w) for c in random_cells(seed, n, w)]
    if name == "malicious":          # reading iii: the scheme-aware worst case
        return pattern("stride" if scheme in ("raw", "ras") else "diagonal", scheme, w, seed, n)
    raise ValueError(name)


PATTERNS = ["contiguous", "stride", "diagonal", "random", "malicious"]
SCHEMES = ["raw", "ras", "rap"]


def sweep(w, seed, first, n_trials):
    """hist[pattern][scheme][c] over trials first .. first+n_trials-1 (nested lists)."""
    h = [[[0] * (w + 1) for _ in SCHEMES] for _ in PATTERNS]
    for n in range(first, first + n_trials):
        P, r = perm(seed, n, w), ras_shifts(seed, n, w)
        for pi, p in enumerate(PATTERNS):
            for si, s in enumerate(SCHEMES):
                h[pi][si][congestion(pattern(p, s, w, seed, n), s, w, P, r)] += 1
    return h
