/*
 * rap_oracle.c -- plain, slow, obviously-correct CPU oracle for the RAP hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  The product path
 * (paper_conf_icppw_nakanomi14_b200/, librap.so) never includes, links or calls it,
 * and this file includes nothing from the product tree.
 *
 * Paper: K. Nakano, S. Matsumae, Y. Ito, "Random Address Permute-Shift Technique for
 * the Shared Memory on GPUs", ICPPW 2014.  Citations "P:L<a>-<b>" are line numbers
 * of /root/reference/PAPER.md (PDF-extracted text) plus the section / figure / table.
 *
 * What is computed (DESIGN.md "Readings" lists every choice the paper leaves open):
 *   O1  Philox4x32-10 (Salmon et al., SC'11) -- the counter-based generator both
 *       sides implement independently (the paper only says "random").
 *   O2  word(seed, n, d, t) = Philox(ctr=(n_lo, n_hi, t>>2, d), key=(seed_lo, seed_hi))[t&3]
 *   O3  P = Durstenfeld shuffle of (0..w-1): for k=w-1..1, j=floor(word(0,w-1-k)*(k+1)/2^32),
 *       swap a[k],a[j]  -- "P selected from all w! permutations uniformly", §IV.
 *   O4  RAS shifts r[i] = floor(word(1,i)*w/2^32) -- independent random r_i, §I.
 *   O5  random-access cells: cell_t = floor(word(2,t)*w^2/2^32), (row,col)=(cell/w, cell%w)
 *       i.i.d. with replacement (Tab.II "Random"; reading ii).
 *   O6  physical address of logical cell (i,j) of a w x w matrix under a scheme:
 *         RAW  i*w + j                         (§III)
 *         RAS  i*w + (j + r[i]) mod w          (§I)
 *         RAP  i*w + (j + P[i]) mod w          (§IV, Fig.6)
 *         PAD  i*(w+1) + j                     (a [w][w+1] array; baseline, not in paper)
 *         XOR  i*w + (j xor i)                 (swizzle baseline, not in paper; w = 2^k)
 *       and the DMM bank of address a is a mod w (§II).
 *   O7  warp access patterns, lane t = 0..w-1 (§III; reading iii/iv):
 *         contiguous (0,t); stride (t,0); diagonal (t,t); random O5;
 *         malicious: RAW,RAS -> (t,0); RAP,XOR -> (t,t); PAD -> (t,(w-t) mod w).
 *   O8  congestion = max over banks of the number of DISTINCT addresses destined to the
 *       bank; identical addresses are merged (§II).
 *   O9  sweep: for n in [first, first+N): O3..O5, then hist[p][s][congestion] += 1.
 *   O10 transpose: dst[c*ld_dst + r] = src[r*ld_src + c], raw bit copy (§III).
 *   O11 RAP layout: phys[i][(j+P[i]) mod w] = logical[i][j] (Fig.6).
 *   O12 DMM time of warps with congestions c_1..c_m: sum(c) + l - 1.
 *
 *   O13 §VII higher-dimensional RAP: a w x w x w x w array, a[i][j][k][l] at
 *       address i*w^3 + j*w^2 + k*w + l, bank l; a scheme stores a[i][j][k][l] at
 *       a[i][j][k][(l + f(i,j,k)) mod w] with
 *         RAW f = 0;  RAS f = r[i][j][k], r = floor(word(1, i*w^2+j*w+k) * w / 2^32);
 *         1P  f = P[k];  R1P f = P[i] + P[j] + P[k];  3P f = P[i] + Q[j] + R[k]
 *       (P, Q, R = Durstenfeld permutations from domains 0, 3, 4 -- reading xiii).
 *       Warp patterns, lane t: contiguous (0,0,0,t); stride1 (0,0,t,0); stride2 (0,t,0,0);
 *       stride3 (t,0,0,0); random: w cells of w^4 i.i.d. with replacement (domain 2);
 *       malicious: RAW, RAS -> stride1; 1P -> stride2; R1P, 3P -> the paper's groups of the 6
 *       permutations of (x, y, z), group g = (3g, 3g+1, 3g+2), l = 0, lanes past
 *       6*floor(w/6) repeat lane 0's request (merged).
 *   O14 data-dependent tile gather (NEXT-4): x_{k+1}[o] = x_k[idx[o]], x_0[o] = o.
 *
 * Every function returns 0 on success and a negative value on a bad argument.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define ORACLE_MAX_W 256

enum { O_RAW = 0, O_RAS = 1, O_RAP = 2, O_PAD = 3, O_XOR = 4, O_NSCHEME = 5 };
enum { O_CONTIGUOUS = 0, O_STRIDE = 1, O_DIAGONAL = 2, O_RANDOM = 3, O_MALICIOUS = 4,
       O_NPATTERN = 5 };
enum { D_FY = 0, D_RAS = 1, D_RANDOM = 2 };

/* ---------------- O1: Philox4x32-10 ---------------- */
void oracle_philox4x32_10(const uint32_t ctr_in[4], const uint32_t key_in[2], uint32_t out[4])
{
    uint32_t c0 = ctr_in[0], c1 = ctr_in[1], c2 = ctr_in[2], c3 = ctr_in[3];
    uint32_t k0 = key_in[0], k1 = key_in[1];
    for (int round = 0; round < 10; ++round) {
        if (round > 0) { k0 += 0x9E3779B9u; k1 += 0xBB67AE85u; }   /* key bump */
        uint64_t p0 = (uint64_t)0xD2511F53u * c0;
        uint64_t p1 = (uint64_t)0xCD9E8D57u * c2;
        uint32_t hi0 = (uint32_t)(p0 >> 32), lo0 = (uint32_t)p0;
        uint32_t hi1 = (uint32_t)(p1 >> 32), lo1 = (uint32_t)p1;
        uint32_t n0 = hi1 ^ c1 ^ k0;
        uint32_t n1 = lo1;
        uint32_t n2 = hi0 ^ c3 ^ k1;
        uint32_t n3 = lo0;
        c0 = n0; c1 = n1; c2 = n2; c3 = n3;
    }
    out[0] = c0; out[1] = c1; out[2] = c2; out[3] = c3;
}

/* ---------------- O2: the counter contract ---------------- */
uint32_t oracle_word(uint64_t seed, uint64_t n, uint32_t d, uint32_t t)
{
    uint32_t ctr[4] = { (uint32_t)n, (uint32_t)(n >> 32), t >> 2, d };
    uint32_t key[2] = { (uint32_t)seed, (uint32_t)(seed >> 32) };
    uint32_t out[4];
    oracle_philox4x32_10(ctr, key, out);
    return out[t & 3u];
}

/* floor(u * m / 2^32): the multiply-shift map of a 32-bit word onto [0, m). */
static uint32_t mulshift(uint32_t u, uint32_t m) { return (uint32_t)(((uint64_t)u * m) >> 32); }

/* ---------------- O3: permutation P (Durstenfeld / Fisher-Yates) ---------------- */
int oracle_perm_domain(uint64_t seed, uint64_t n, uint32_t w, uint32_t d, uint32_t *a)
{
    if (w < 1 || w > ORACLE_MAX_W || !a) return -1;
    for (uint32_t i = 0; i < w; ++i) a[i] = i;
    for (uint32_t k = w - 1; k >= 1; --k) {
        uint32_t u = oracle_word(seed, n, d, w - 1 - k);
        uint32_t j = mulshift(u, k + 1);
        uint32_t tmp = a[k]; a[k] = a[j]; a[j] = tmp;
    }
    return 0;
}

int oracle_perm(uint64_t seed, uint64_t n, uint32_t w, uint32_t *a)
{
    return oracle_perm_domain(seed, n, w, D_FY, a);
}

/* ---------------- O4: RAS shift vector ---------------- */
int oracle_ras_shifts(uint64_t seed, uint64_t n, uint32_t w, uint32_t *r)
{
    if (w < 1 || w > ORACLE_MAX_W || !r) return -1;
    for (uint32_t i = 0; i < w; ++i) r[i] = mulshift(oracle_word(seed, n, D_RAS, i), w);
    return 0;
}

/* ---------------- O5: random-access cells ---------------- */
int oracle_random_cells(uint64_t seed, uint64_t n, uint32_t w, uint32_t *rows, uint32_t *cols)
{
    if (w < 1 || w > ORACLE_MAX_W || !rows || !cols) return -1;
    for (uint32_t t = 0; t < w; ++t) {
        uint32_t cell = mulshift(oracle_word(seed, n, D_RANDOM, t), w * w);
        rows[t] = cell / w;
        cols[t] = cell % w;
    }
    return 0;
}

/* ---------------- O6: address maps and the DMM bank ---------------- */
static int is_pow2(uint32_t w) { return w && !(w & (w - 1)); }

/* Physical address of logical cell (i,j); shift = r (RAS) or P (RAP), unused otherwise. */
int64_t oracle_address(uint32_t scheme, uint32_t w, uint32_t i, uint32_t j, const uint32_t *shift)
{
    if (i >= w || j >= w) return -1;
    switch (scheme) {
    case O_RAW: return (int64_t)i * w + j;
    case O_RAS:
    case O_RAP: if (!shift) return -1; return (int64_t)i * w + (j + shift[i]) % w;
    case O_PAD: return (int64_t)i * (w + 1) + j;
    case O_XOR: if (!is_pow2(w)) return -1; return (int64_t)i * w + (j ^ i);
    default: return -1;
    }
}

/* ---------------- O8: congestion of one warp access ---------------- */
int oracle_congestion(uint32_t w, uint32_t n, const uint32_t *rows, const uint32_t *cols,
                      uint32_t scheme, const uint32_t *shift, uint32_t *congestion_out)
{
    if (w < 1 || w > ORACLE_MAX_W || n > ORACLE_MAX_W || !congestion_out) return -1;
    int64_t addr[ORACLE_MAX_W];
    for (uint32_t t = 0; t < n; ++t) {
        addr[t] = oracle_address(scheme, w, rows[t], cols[t], shift);
        if (addr[t] < 0) return -1;
    }
    /* count, per bank, the distinct addresses: request t is counted only if no earlier
       request carries the same address (merged requests). */
    uint32_t count[ORACLE_MAX_W];
    memset(count, 0, sizeof(count));
    for (uint32_t t = 0; t < n; ++t) {
        int duplicate = 0;
        for (uint32_t s = 0; s < t; ++s)
            if (addr[s] == addr[t]) { duplicate = 1; break; }
        if (!duplicate) count[addr[t] % w] += 1;
    }
    uint32_t c = 0;
    for (uint32_t b = 0; b < w; ++b)
        if (count[b] > c) c = count[b];
    *congestion_out = c;
    return 0;
}

/* ---------------- O7: warp access patterns ---------------- */
int oracle_pattern_cells(uint32_t pattern, uint32_t scheme, uint32_t w, uint64_t seed, uint64_t n,
                         uint32_t *rows, uint32_t *cols)
{
    if (w < 1 || w > ORACLE_MAX_W || !rows || !cols || scheme >= O_NSCHEME) return -1;
    if (pattern == O_MALICIOUS) {
        /* reading iii: the adversary knows the scheme, not P or r */
        switch (scheme) {
        case O_RAW: case O_RAS: pattern = O_STRIDE; break;
        case O_RAP: case O_XOR: pattern = O_DIAGONAL; break;
        case O_PAD:
            for (uint32_t t = 0; t < w; ++t) { rows[t] = t; cols[t] = (w - t) % w; }
            return 0;
        }
    }
    switch (pattern) {
    case O_CONTIGUOUS: for (uint32_t t = 0; t < w; ++t) { rows[t] = 0; cols[t] = t; } return 0;
    case O_STRIDE:     for (uint32_t t = 0; t < w; ++t) { rows[t] = t; cols[t] = 0; } return 0;
    case O_DIAGONAL:   for (uint32_t t = 0; t < w; ++t) { rows[t] = t; cols[t] = t; } return 0;
    case O_RANDOM:     return oracle_random_cells(seed, n, w, rows, cols);
    default: return -1;
    }
}

/* ---------------- O9: the Monte-Carlo sweep ---------------- */
static uint32_t popcount5(uint32_t m) { uint32_t c = 0; for (int b = 0; b < 5; ++b) c += (m >> b) & 1u; return c; }

static int sweep_range(uint32_t w, uint32_t pattern_mask, uint32_t scheme_mask, uint64_t seed,
                       uint64_t first, uint64_t count, uint64_t *hist)
{
    const uint32_t ns = popcount5(scheme_mask);
    uint32_t P[ORACLE_MAX_W], r[ORACLE_MAX_W], rows[ORACLE_MAX_W], cols[ORACLE_MAX_W];
    for (uint64_t k = 0; k < count; ++k) {
        uint64_t n = first + k;
        oracle_perm(seed, n, w, P);
        oracle_ras_shifts(seed, n, w, r);
        uint32_t pi = 0;
        for (uint32_t p = 0; p < O_NPATTERN; ++p) {
            if (!((pattern_mask >> p) & 1u)) continue;
            uint32_t si = 0;
            for (uint32_t s = 0; s < O_NSCHEME; ++s) {
                if (!((scheme_mask >> s) & 1u)) continue;
                if (oracle_pattern_cells(p, s, w, seed, n, rows, cols)) return -1;
                const uint32_t *shift = (s == O_RAS) ? r : (s == O_RAP) ? P : NULL;
                uint32_t c;
                if (oracle_congestion(w, w, rows, cols, s, shift, &c)) return -1;
                hist[((uint64_t)pi * ns + si) * (w + 1) + c] += 1;
                ++si;
            }
            ++pi;
        }
    }
    return 0;
}

/* hist: u64[popcount(pattern_mask)][popcount(scheme_mask)][w+1], ACCUMULATED (+=). */
int oracle_sweep(uint32_t w, uint32_t pattern_mask, uint32_t scheme_mask, uint64_t seed,
                 uint64_t first, uint64_t n_trials, uint64_t *hist, int threads)
{
    if (w < 2 || w > ORACLE_MAX_W || !hist) return -1;
    if (pattern_mask == 0 || pattern_mask > 31 || scheme_mask == 0 || scheme_mask > 31) return -1;
    if (((scheme_mask >> O_XOR) & 1u) && !is_pow2(w)) return -1;
    const size_t nbins = (size_t)popcount5(pattern_mask) * popcount5(scheme_mask) * (w + 1);
    if (threads < 1) threads = 1;
    uint64_t *part = (uint64_t *)calloc((size_t)threads * nbins, sizeof(uint64_t));
    if (!part) return -2;
    int err = 0;
#ifdef _OPENMP
#pragma omp parallel for num_threads(threads) schedule(static) reduction(|:err)
#endif
    for (int th = 0; th < threads; ++th) {
        uint64_t lo = n_trials * (uint64_t)th / (uint64_t)threads;
        uint64_t hi = n_trials * (uint64_t)(th + 1) / (uint64_t)threads;
        err |= sweep_range(w, pattern_mask, scheme_mask, seed, first + lo, hi - lo,
                           part + (size_t)th * nbins);
    }
    for (int th = 0; th < threads; ++th)
        for (size_t b = 0; b < nbins; ++b) hist[b] += part[(size_t)th * nbins + b];
    free(part);
    return err ? -1 : 0;
}

/* ---------------- O10: the transpose ---------------- */
int oracle_transpose(const void *src, void *dst, int64_t rows, int64_t cols, int64_t ld_src,
                     int64_t ld_dst, uint32_t elem_bytes, int threads)
{
    if (rows < 0 || cols < 0 || ld_src < cols || ld_dst < rows) return -1;
    if (elem_bytes != 1 && elem_bytes != 2 && elem_bytes != 4 && elem_bytes != 8) return -1;
    if ((rows && cols) && (!src || !dst)) return -1;
    if (threads < 1) threads = 1;
    const unsigned char *s = (const unsigned char *)src;
    unsigned char *d = (unsigned char *)dst;
#ifdef _OPENMP
#pragma omp parallel for num_threads(threads) schedule(static)
#endif
    for (int64_t r = 0; r < rows; ++r)
        for (int64_t c = 0; c < cols; ++c)
            memcpy(d + (size_t)(c * ld_dst + r) * elem_bytes,
                   s + (size_t)(r * ld_src + c) * elem_bytes, elem_bytes);
    return 0;
}

/* ---------------- O11: RAP layout of a w x w matrix ---------------- */
int oracle_rap_layout(uint32_t w, const uint32_t *P, const uint32_t *logical, uint32_t *phys)
{
    if (w < 1 || w > ORACLE_MAX_W || !P || !logical || !phys) return -1;
    for (uint32_t i = 0; i < w; ++i)
        for (uint32_t j = 0; j < w; ++j)
            phys[i * w + (j + P[i]) % w] = logical[i * w + j];
    return 0;
}

/* ---------------- O12: DMM time of a sequence of warp accesses ---------------- */
int64_t oracle_dmm_time(const uint32_t *congestion, uint32_t m, uint32_t latency)
{
    if (!congestion || m == 0 || latency < 1) return -1;
    int64_t stages = 0;
    for (uint32_t i = 0; i < m; ++i) stages += congestion[i];
    return stages + latency - 1;
}

/* ---------------- O13: higher-dimensional RAP (w^4 arrays) ---------------- */
enum { S4_RAW = 0, S4_RAS = 1, S4_1P = 2, S4_R1P = 3, S4_3P = 4, S4_N = 5 };
enum { P4_CONTIGUOUS = 0, P4_STRIDE1 = 1, P4_STRIDE2 = 2, P4_STRIDE3 = 3, P4_RANDOM = 4,
       P4_MALICIOUS = 5, P4_N = 6 };
enum { D_Q = 3, D_R = 4 };

/* shift f(i,j,k) of a scheme; P, Q, R given, RAS shifts drawn from the counter contract */
int64_t oracle_shift4(uint32_t scheme, uint32_t w, uint32_t i, uint32_t j, uint32_t k,
                      const uint32_t *P, const uint32_t *Q, const uint32_t *R, uint64_t seed, uint64_t n)
{
    if (i >= w || j >= w || k >= w) return -1;
    switch (scheme) {
    case S4_RAW: return 0;
    case S4_RAS: return mulshift(oracle_word(seed, n, D_RAS, (i * w + j) * w + k), w);
    case S4_1P: return P[k];
    case S4_R1P: return ((uint64_t)P[i] + P[j] + P[k]) % w;
    case S4_3P: return ((uint64_t)P[i] + Q[j] + R[k]) % w;
    default: return -1;
    }
}

/* physical address of a[i][j][k][l] */
int64_t oracle_address4(uint32_t scheme, uint32_t w, uint32_t i, uint32_t j, uint32_t k, uint32_t l,
                        const uint32_t *P, const uint32_t *Q, const uint32_t *R, uint64_t seed, uint64_t n)
{
    if (l >= w) return -1;
    int64_t f = oracle_shift4(scheme, w, i, j, k, P, Q, R, seed, n);
    if (f < 0) return -1;
    int64_t w2 = (int64_t)w * w;
    return ((int64_t)i * w2 + (int64_t)j * w) * w + (int64_t)k * w + (l + f) % w;
}

/* congestion of n requests to cells (i,j,k,l): distinct addresses per bank (address mod w) */
int oracle_congestion4(uint32_t w, uint32_t nreq, const uint32_t *ci, const uint32_t *cj, const uint32_t *ck,
                       const uint32_t *cl, uint32_t scheme, const uint32_t *P, const uint32_t *Q,
                       const uint32_t *R, uint64_t seed, uint64_t n, uint32_t *congestion_out)
{
    if (w < 1 || w > ORACLE_MAX_W || nreq > ORACLE_MAX_W || !congestion_out) return -1;
    int64_t addr[ORACLE_MAX_W];
    for (uint32_t t = 0; t < nreq; ++t) {
        addr[t] = oracle_address4(scheme, w, ci[t], cj[t], ck[t], cl[t], P, Q, R, seed, n);
        if (addr[t] < 0) return -1;
    }
    uint32_t count[ORACLE_MAX_W];
    memset(count, 0, sizeof(count));
    for (uint32_t t = 0; t < nreq; ++t) {
        int duplicate = 0;
        for (uint32_t s = 0; s < t; ++s)
            if (addr[s] == addr[t]) { duplicate = 1; break; }
        if (!duplicate) count[addr[t] % w] += 1;
    }
    uint32_t c = 0;
    for (uint32_t b = 0; b < w; ++b)
        if (count[b] > c) c = count[b];
    *congestion_out = c;
    return 0;
}

int oracle_pattern4(uint32_t pattern, uint32_t scheme, uint32_t w, uint64_t seed, uint64_t n,
                    uint32_t *ci, uint32_t *cj, uint32_t *ck, uint32_t *cl)
{
    if (w < 1 || w > 255 || scheme >= S4_N) return -1;
    if (pattern == P4_MALICIOUS) {
        if (scheme == S4_RAW || scheme == S4_RAS) pattern = P4_STRIDE1;
        else if (scheme == S4_1P) pattern = P4_STRIDE2;
        else {
            /* the 6 permutations of (x, y, z) = (3g, 3g+1, 3g+2) share f under R1P */
            uint32_t groups = w / 6;
            for (uint32_t t = 0; t < w; ++t) {
                uint32_t g = t / 6, m = t % 6;
                if (g >= groups || 3 * g + 2 >= w) { g = 0; m = 0; }
                uint32_t x = 3 * g, y = 3 * g + 1, z = 3 * g + 2;
                static const int perm6[6][3] = {{0, 1, 2}, {0, 2, 1}, {1, 0, 2}, {1, 2, 0}, {2, 0, 1}, {2, 1, 0}};
                uint32_t v[3] = {x, y, z};
                ci[t] = v[perm6[m][0]]; cj[t] = v[perm6[m][1]]; ck[t] = v[perm6[m][2]]; cl[t] = 0;
            }
            return 0;
        }
    }
    for (uint32_t t = 0; t < w; ++t) {
        ci[t] = cj[t] = ck[t] = cl[t] = 0;
        switch (pattern) {
        case P4_CONTIGUOUS: cl[t] = t; break;
        case P4_STRIDE1: ck[t] = t; break;
        case P4_STRIDE2: cj[t] = t; break;
        case P4_STRIDE3: ci[t] = t; break;
        case P4_RANDOM: {
            uint64_t w4 = (uint64_t)w * w * w * w;
            uint32_t cell = (uint32_t)(((uint64_t)oracle_word(seed, n, D_RANDOM, t) * w4) >> 32);
            cl[t] = cell % w; cell /= w;
            ck[t] = cell % w; cell /= w;
            cj[t] = cell % w; cell /= w;
            ci[t] = cell;
            break;
        }
        default: return -1;
        }
    }
    return 0;
}

static int sweep4_range(uint32_t w, uint32_t pattern_mask, uint32_t scheme_mask, uint64_t seed,
                        uint64_t first, uint64_t count, uint64_t *hist)
{
    const uint32_t ns = __builtin_popcount(scheme_mask);
    uint32_t P[ORACLE_MAX_W], Q[ORACLE_MAX_W], R[ORACLE_MAX_W];
    uint32_t ci[ORACLE_MAX_W], cj[ORACLE_MAX_W], ck[ORACLE_MAX_W], cl[ORACLE_MAX_W];
    for (uint64_t q = 0; q < count; ++q) {
        uint64_t n = first + q;
        oracle_perm_domain(seed, n, w, D_FY, P);
        oracle_perm_domain(seed, n, w, D_Q, Q);
        oracle_perm_domain(seed, n, w, D_R, R);
        uint32_t pi = 0;
        for (uint32_t p = 0; p < P4_N; ++p) {
            if (!((pattern_mask >> p) & 1u)) continue;
            uint32_t si = 0;
            for (uint32_t sc = 0; sc < S4_N; ++sc) {
                if (!((scheme_mask >> sc) & 1u)) continue;
                uint32_t c;
                if (oracle_pattern4(p, sc, w, seed, n, ci, cj, ck, cl)) return -1;
                if (oracle_congestion4(w, w, ci, cj, ck, cl, sc, P, Q, R, seed, n, &c)) return -1;
                hist[((uint64_t)pi * ns + si) * (w + 1) + c] += 1;
                ++si;
            }
            ++pi;
        }
    }
    return 0;
}

/* hist: u64[popcount(pattern_mask)][popcount(scheme_mask)][w+1], ACCUMULATED */
int oracle_sweep4(uint32_t w, uint32_t pattern_mask, uint32_t scheme_mask, uint64_t seed,
                  uint64_t first, uint64_t n_trials, uint64_t *hist, int threads)
{
    if (w < 2 || w > 64 || !hist) return -1;
    if (pattern_mask == 0 || pattern_mask > 63 || scheme_mask == 0 || scheme_mask > 31) return -1;
    const size_t nbins = (size_t)__builtin_popcount(pattern_mask) * __builtin_popcount(scheme_mask) * (w + 1);
    if (threads < 1) threads = 1;
    uint64_t *part = (uint64_t *)calloc((size_t)threads * nbins, sizeof(uint64_t));
    if (!part) return -2;
    int err = 0;
#ifdef _OPENMP
#pragma omp parallel for num_threads(threads) schedule(static) reduction(|:err)
#endif
    for (int th = 0; th < threads; ++th) {
        uint64_t lo = n_trials * (uint64_t)th / (uint64_t)threads;
        uint64_t hi = n_trials * (uint64_t)(th + 1) / (uint64_t)threads;
        err |= sweep4_range(w, pattern_mask, scheme_mask, seed, first + lo, hi - lo, part + (size_t)th * nbins);
    }
    for (int th = 0; th < threads; ++th)
        for (size_t b = 0; b < nbins; ++b) hist[b] += part[(size_t)th * nbins + b];
    free(part);
    return err ? -1 : 0;
}

/* ---------------- O14: data-dependent tile gather (NEXT-4) ---------------- */
/* out = in composed `reps` times with the gather idx: x_{k+1}[o] = x_k[idx[o]], x_0[o] = o */
int oracle_gather_power(const uint16_t *idx, uint32_t n, uint32_t reps, uint32_t *out)
{
    if (!idx || !out || n == 0 || n > 65536) return -1;
    uint32_t *tmp = (uint32_t *)malloc((size_t)n * sizeof(uint32_t));
    if (!tmp) return -2;
    for (uint32_t o = 0; o < n; ++o) { if (idx[o] >= n) { free(tmp); return -1; } out[o] = o; }
    for (uint32_t k = 0; k < reps; ++k) {
        for (uint32_t o = 0; o < n; ++o) tmp[o] = out[idx[o]];
        memcpy(out, tmp, (size_t)n * sizeof(uint32_t));
    }
    free(tmp);
    return 0;
}

int oracle_max_threads(void)
{
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}
