// congestion.cu -- steps C1-C4 of the RAP hot path: the DMM congestion evaluator and its
// Monte-Carlo sweep (Table II, §V), plus the batched evaluator,
// the trace evaluator and the device permutation generator (T0).
//
// One CUDA warp simulates one DMM warp of w <= 32 threads (§II): lane t issues the
// request of DMM thread t.  Congestion: requests to the same address are merged
// (one leader per address), then lane v counts the distinct requests to bank v from five
// 32-bit bank-bit masks (rap_warp.cuh) and the congestion is the warp maximum
// (__reduce_max_sync).  The default sweep (sweep32_kernel / sweep_kernel) draws each trial's
// permutation in lane mode as 5 bit planes; the ablation kernel (sweep_match_kernel) keeps the
// north-star sketch: warp Fisher-Yates by __shfl_sync and __match_any_sync histograms.
// Histograms: shared-memory u32 counters (evaluation e counted by lane e), reduced per CTA and
// added once to the caller's u64 bins.
#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>

#include "rap_rng.cuh"
#include "rap_warp.cuh"
#include "rap_internal.h"

namespace rapk {

constexpr int kSweepWarps = 8;
constexpr int kMaxEval = 25;                 // 5 patterns x 5 schemes
constexpr int kMaxBins = kMaxEval * (RAP_MAX_W + 1);

// Bank of logical cell (row, col) under `scheme`; sh = shift of that row (r[row] or P[row]).
__device__ __forceinline__ uint32_t bank_of(int scheme, uint32_t row, uint32_t col, uint32_t sh, uint32_t w) {
    switch (scheme) {
    case RAP_SCHEME_RAS:
    case RAP_SCHEME_RAP: { const uint32_t b = col + sh; return b >= w ? b - w : b; }
    case RAP_SCHEME_PAD: { const uint32_t b = row + col; return b >= w ? b - w : b; }
    case RAP_SCHEME_XOR: return col ^ row;
    default: return col;
    }
}

// Generic evaluator: lane t (< w) requests (row, col); P / r: lane i holds P[i] / r[i].
__device__ __forceinline__ uint32_t warp_congestion(uint32_t row, uint32_t col, int scheme, uint32_t P,
                                                    uint32_t r, uint32_t lane, uint32_t w,
                                                    const LaneSel &ls) {
    const uint32_t active = (w >= 32) ? kFull : ((1u << w) - 1u);
    uint32_t sh = 0;
    if (scheme == RAP_SCHEME_RAS || scheme == RAP_SCHEME_RAP)
        sh = __shfl_sync(kFull, scheme == RAP_SCHEME_RAP ? P : r, row & 31u);
    const uint32_t bank = bank_of(scheme, row, col, sh, w);
    const uint32_t counted = first_occurrences(row * 32u + col, active, lane);
    return max_bank_load(bank, counted, ls);
}

// ---------------------------------------------------------------------------------------
// Ablation variant (the north-star sketch): __match_any_sync on the address to merge, then
// popc(__match_any_sync(bank)).  Bit-identical results; kept to measure the design choice.
template <int W>
__device__ __forceinline__ uint32_t warp_congestion_match(uint32_t row, uint32_t col, int scheme, uint32_t P,
                                                          uint32_t r, uint32_t lane, uint32_t w_rt,
                                                          bool dedupe) {
    const uint32_t w = W ? (uint32_t)W : w_rt;
    const bool active = lane < w;
    uint32_t sh = 0;
    if (scheme == RAP_SCHEME_RAS || scheme == RAP_SCHEME_RAP)
        sh = __shfl_sync(kFull, scheme == RAP_SCHEME_RAP ? P : r, row & 31u);
    const uint32_t bank = bank_of(scheme, row, col, sh, w);
    const uint32_t addr = row * 32u + col;
    uint32_t key = bank;
    if (dedupe) {                                        // merge identical addresses
        const uint32_t same = __match_any_sync(kFull, active ? addr : (0x40000000u | lane));
        const bool leader = (uint32_t)(__ffs(same) - 1) == lane;
        key = leader ? bank : (0x10000u | lane);
    }
    if (!active) key = 0x20000u | lane;
    const uint32_t cnt = __popc(__match_any_sync(kFull, key));
    return __reduce_max_sync(kFull, cnt);
}

// Cells of lane t for a built-in pattern (reading iii for malicious).
__device__ __forceinline__ void pattern_cell(int pattern, int scheme, uint32_t lane, uint32_t w,
                                             uint32_t rrow, uint32_t rcol, uint32_t &row, uint32_t &col) {
    switch (pattern) {
    case RAP_PAT_CONTIGUOUS: row = 0; col = lane; break;
    case RAP_PAT_STRIDE: row = lane; col = 0; break;
    case RAP_PAT_DIAGONAL: row = lane; col = lane; break;
    case RAP_PAT_RANDOM: row = rrow; col = rcol; break;
    default:  // malicious, scheme-aware
        if (scheme == RAP_SCHEME_RAW || scheme == RAP_SCHEME_RAS) { row = lane; col = 0; }
        else if (scheme == RAP_SCHEME_PAD) { row = lane; col = (lane == 0) ? 0u : w - lane; }
        else { row = lane; col = lane; }
        break;
    }
}

// Flush the per-warp u32 histograms of this CTA into the caller's u64 bins.
__device__ __forceinline__ void flush_hist(uint32_t (*sh)[kMaxBins], int nwarps, uint32_t nbins,
                                           uint64_t *hist) {
    __syncthreads();
    for (uint32_t b = threadIdx.x; b < nbins; b += blockDim.x) {
        uint64_t s = 0;
        for (int k = 0; k < nwarps; ++k) s += sh[k][b];
        if (s) atomicAdd((unsigned long long *)(hist + b), (unsigned long long)s);
    }
}

// ------------------------------------------------------------------ C1-C4 sweep (default)
// Two phases per batch of 32 trials, per warp:
//  lane mode  (lane L <-> trial n0+L): the lane draws its own Philox words (C1), runs the
//             whole Durstenfeld shuffle on a bit-sliced permutation held in 5 registers --
//             plane k has bit i = bit k of a[i], so a swap a[k] <-> a[j] is a few shifts and
//             XORs per plane, no shuffles (C2) -- and stores its RAS shifts and random cells
//             into a [32][33] shared-memory transpose buffer (+1 padding: the lane-mode write
//             and the warp-mode read are both conflict-free).
//  warp mode  (lane t <-> DMM thread t of trial n0+m, m = 0..31): broadcast trial m's planes
//             (5 shuffles), unpack P[t]; read r[t] and cell t from shared memory; evaluate
//             every selected (pattern, scheme) with the ballot evaluator (C3); lane e counts
//             evaluation e in the CTA histogram (C4).
// launch shape of the default sweep (measured on B200, profiles/r01_tune_sweep.txt,
// r02_ab_sweep*.txt): 4-warp CTAs, 8 per SM (64 registers; with the ballot evaluator 7 CTAs at
// 73 registers were 2.9 % faster, with the shared-memory bank counters 8 CTAs are 1.2 % faster),
// and a grid of 16 x the resident CTAs so that SMs that finish early pick up more work (+11%
// over one persistent wave).  The macros exist for tuning
// builds (RAP_EXTRA_NVCC_FLAGS)
#ifndef RAP_SWEEP_WARPS
#define RAP_SWEEP_WARPS 4
#endif
#ifndef RAP_SWEEP_MINB
#define RAP_SWEEP_MINB 8
#endif
#ifndef RAP_SWEEP_GRID_MULT
#define RAP_SWEEP_GRID_MULT 16
#endif
constexpr int kSweepWarpsV2 = RAP_SWEEP_WARPS;

// RAP_SWEEP_SWAP_MULHI (ablation, default 0): in the plane swap, pl >> d on the FMA pipe as
// umulhi(pl, 2^(32-d)) (IMAD.HI): 3.9 ALU instructions fewer per trial for the ALU-bound sweep,
// yet 2 % slower (4.689 vs 4.768 G trials/s, profiles/r02c_ab_sweep_mulhi.txt).  d = 0 (j = k, no
// swap) makes the multiplier 2^32 -> 0 in PTX's shl, so y = pl & mj, and pl ^= y ^ (y * 1)
// leaves pl unchanged as it must.  Bit-identical.
#ifndef RAP_SWEEP_SWAP_MULHI
#define RAP_SWEEP_SWAP_MULHI 0
#endif
template <int W>
__device__ __forceinline__ void swap_planes(uint32_t (&pl)[5], uint32_t k, uint32_t j) {
    // j <= k: y holds bit_j ^ bit_k at position j; flipping bits j and k by y swaps them.
    // y << d runs on the FMA pipe as y * 2^d (the sweep is bound by the ALU pipe); 2^d is made
    // in PTX so that the compiler does not turn the multiply back into a shift.
    const uint32_t d = k - j, mj = 1u << j;
    uint32_t sd;
    asm("shl.b32 %0, %1, %2;" : "=r"(sd) : "r"(1u), "r"(d));
#if RAP_SWEEP_SWAP_MULHI
    uint32_t sr;                                          // 2^(32-d); 0 for d = 0 (shl clamps)
    asm("shl.b32 %0, %1, %2;" : "=r"(sr) : "r"(1u), "r"(32u - d));
#pragma unroll
    for (int b = 0; b < 5; ++b) {
        uint32_t hi;
        asm("mul.hi.u32 %0, %1, %2;" : "=r"(hi) : "r"(pl[b]), "r"(sr));
        const uint32_t y = (pl[b] ^ hi) & mj;
        pl[b] ^= y ^ (y * sd);
    }
#else
#pragma unroll
    for (int b = 0; b < 5; ++b) {
        const uint32_t y = (pl[b] ^ (pl[b] >> d)) & mj;
        pl[b] ^= y ^ (y * sd);
    }
#endif
}

// C1+C2 in lane mode: P_n = perm(seed, n, w) as bit planes.
template <int W>
__device__ __forceinline__ void lane_perm_planes(uint64_t seed, uint64_t n, uint32_t w_rt, uint32_t (&pl)[5]) {
    const uint32_t w = W ? (uint32_t)W : w_rt;
    pl[0] = 0xAAAAAAAAu; pl[1] = 0xCCCCCCCCu; pl[2] = 0xF0F0F0F0u; pl[3] = 0xFF00FF00u; pl[4] = 0xFFFF0000u;
    if (W) {
#pragma unroll
        for (int blk = 0; blk < (W ? (W + 2) / 4 : 1); ++blk) {
            const uint4 c = philox_block(seed, n, kDomainFY, blk);
            const uint32_t u[4] = {c.x, c.y, c.z, c.w};
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                const int t = 4 * blk + i;
                if (t >= W - 1) break;
                const uint32_t k = (uint32_t)(W - 1 - t);
                swap_planes<W>(pl, k, mulshift(u[i], k + 1));
            }
        }
    } else {
        for (uint32_t blk = 0; 4 * blk + 1 < w; ++blk) {
            const uint4 c = philox_block(seed, n, kDomainFY, blk);
            const uint32_t u[4] = {c.x, c.y, c.z, c.w};
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                const uint32_t t = 4 * blk + i;
                if (t + 1 < w) {
                    const uint32_t k = w - 1 - t;
                    swap_planes<0>(pl, k, mulshift(u[i], k + 1));
                }
            }
        }
    }
}

__device__ __forceinline__ uint32_t plane_value(const uint32_t (&q)[5], uint32_t i) {
    uint32_t v = 0;
#pragma unroll
    for (int b = 0; b < 5; ++b) v |= ((q[b] >> i) & 1u) << b;
    return v;
}
__device__ __forceinline__ uint32_t plane_value4(const uint32_t (&q)[5], uint32_t i) {   // 4 * value
    uint32_t v = 0;
#pragma unroll
    for (int b = 0; b < 5; ++b) v |= ((q[b] >> i) & 1u) << (b + 2);
    return v;
}

// (x mod w) for x < 2w; a mask when w is a compile-time power of two
template <int W>
__device__ __forceinline__ uint32_t mod_w(uint32_t x, uint32_t w) {
    if (W && !(W & (W - 1))) return x & (uint32_t)(W - 1);
    return x >= w ? x - w : x;
}

// RAP_SWEEP_GENERIC_DEDUP (default 1): the w < 32 kernel finds the merged requests of the random
// access with a per-warp cell bitmap and one atom.shared.or (as sweep32_kernel's
// RAP_SWEEP_DEDUP_SMEM) instead of __match_any_sync
#ifndef RAP_SWEEP_GENERIC_DEDUP
#define RAP_SWEEP_GENERIC_DEDUP 1
#endif
// PM / SM: pattern / scheme masks fixed at compile time (0 = take the runtime masks), so the
// common configurations evaluate with no mask tests and constant evaluation slots.
template <int W, uint32_t PM, uint32_t SM>
__global__ void __launch_bounds__(kSweepWarpsV2 * 32)
sweep_kernel(uint32_t w_rt, uint32_t pmask_rt, uint32_t smask_rt, uint64_t seed, uint64_t first,
             uint64_t n_trials, uint64_t *__restrict__ hist) {
    const uint32_t w = W ? (uint32_t)W : w_rt;
    const uint32_t pmask = PM ? PM : pmask_rt, smask = SM ? SM : smask_rt;
    __shared__ uint32_t sh_hist[kMaxBins];
    __shared__ uint32_t sh_tr[kSweepWarpsV2][32 * 33];
    __shared__ uint32_t sh_bm[RAP_SWEEP_GENERIC_DEDUP ? kSweepWarpsV2 : 1][32];   // cell bitmap, row words
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    const uint32_t npat = __popc(pmask), nsch = __popc(smask);
    const uint32_t nbins = npat * nsch * (w + 1);
    for (uint32_t b = threadIdx.x; b < nbins; b += blockDim.x) sh_hist[b] = 0;
    if (RAP_SWEEP_GENERIC_DEDUP) sh_bm[RAP_SWEEP_GENERIC_DEDUP ? warp : 0][lane] = 0u;
    __syncthreads();

    const LaneSel ls(lane);
    const uint32_t active = (w >= 32) ? kFull : ((1u << w) - 1u);
    const bool any_random = (pmask >> RAP_PAT_RANDOM) & 1u;
    const bool need_r = ((smask >> RAP_SCHEME_RAS) & 1u) != 0u;
    uint32_t *tr = sh_tr[warp];

    const uint64_t nbatch = (n_trials + 31) / 32;
    const uint64_t stride = (uint64_t)gridDim.x * kSweepWarpsV2;
    for (uint64_t bt = (uint64_t)blockIdx.x * kSweepWarpsV2 + warp; bt < nbatch; bt += stride) {
        const uint64_t n0 = first + bt * 32;
        const uint32_t nvalid = (uint32_t)min((uint64_t)32, n_trials - bt * 32);
        // ---- lane mode: trial n0 + lane
        uint32_t pl[5];
        lane_perm_planes<W>(seed, n0 + lane, w, pl);
        if (need_r || any_random) {
#pragma unroll
            for (int blk = 0; blk < 8; ++blk) {
                if (!W && 4u * blk >= w) break;
                const uint4 cr = need_r ? philox_block(seed, n0 + lane, kDomainRAS, blk) : make_uint4(0, 0, 0, 0);
                const uint4 cc = any_random ? philox_block(seed, n0 + lane, kDomainRandom, blk) : make_uint4(0, 0, 0, 0);
                const uint32_t ur[4] = {cr.x, cr.y, cr.z, cr.w};
                const uint32_t uc[4] = {cc.x, cc.y, cc.z, cc.w};
#pragma unroll
                for (int i = 0; i < 4; ++i) {
                    const uint32_t t = 4 * blk + i;
                    if (W || t < w)
                        tr[t * 33 + lane] = (mulshift(ur[i], w) << 10) | mulshift(uc[i], w * w);
                }
            }
        }
        __syncwarp();
        // ---- warp mode: lane t is DMM thread t of trial n0 + m
        for (uint32_t m = 0; m < nvalid; ++m) {
            uint32_t q[5];
#pragma unroll
            for (int b = 0; b < 5; ++b) q[b] = __shfl_sync(kFull, pl[b], m);
            const uint32_t Pt = plane_value(q, lane);          // P[t]
            const uint32_t P0 = plane_value(q, 0);             // P[0] (uniform)
            const uint32_t packed = (W || lane < w) ? tr[lane * 33 + m] : 0u;
            const uint32_t rt = packed >> 10;                  // r[t]
            const uint32_t r0 = __shfl_sync(kFull, rt, 0);
            uint32_t rrow = 0, rcol = 0, Pr = 0, rr = 0, leaders = active;
            if (any_random) {
                const uint32_t cell = packed & 1023u;
                if (W == 32) { rrow = cell >> 5; rcol = cell & 31u; }
                else { rrow = cell / w; rcol = cell - rrow * w; }
                Pr = plane_value(q, rrow);                     // P[row_t]
                rr = __shfl_sync(kFull, rt, rrow);             // r[row_t]
#if RAP_SWEEP_GENERIC_DEDUP
                {   // merged requests: the lane whose atom.shared.or sets its cell's bit leads
                    uint32_t *bm = sh_bm[RAP_SWEEP_GENERIC_DEDUP ? warp : 0];
                    const bool act = W || lane < w;
                    const uint32_t bit = 1u << rcol;
                    const bool lead = act && !(atomicOr(&bm[rrow], bit) & bit);
                    leaders = __ballot_sync(kFull, lead);
                    __syncwarp();
                    if (act) bm[rrow] = 0u;                    // cleared for the next trial
                    __syncwarp();
                }
#else
                leaders = first_occurrences(rrow * 32u + rcol, active, lane);
#endif
            }
            uint32_t mine = 0, e = 0;
            uint32_t c_stride[5] = {0, 0, 0, 0, 0}, c_diag[5] = {0, 0, 0, 0, 0};
#pragma unroll
            for (int p = 0; p < 5; ++p) {
                if (!((pmask >> p) & 1u)) continue;
#pragma unroll
                for (int s = 0; s < 5; ++s) {
                    if (!((smask >> s) & 1u)) continue;
                    uint32_t c;
                    // malicious (reading iii) is the stride set under RAW/RAS and the diagonal
                    // set under RAP/XOR: the same access, so its evaluation is reused
                    if (p == RAP_PAT_MALICIOUS && (s == RAP_SCHEME_RAW || s == RAP_SCHEME_RAS) &&
                        ((pmask >> RAP_PAT_STRIDE) & 1u)) {
                        c = c_stride[s];
                    } else if (p == RAP_PAT_MALICIOUS && (s == RAP_SCHEME_RAP || s == RAP_SCHEME_XOR) &&
                               ((pmask >> RAP_PAT_DIAGONAL) & 1u)) {
                        c = c_diag[s];
                    } else {
                        uint32_t row, col, shP, shR;
                        switch (p) {
                        case RAP_PAT_CONTIGUOUS: row = 0; col = lane; shP = P0; shR = r0; break;
                        case RAP_PAT_STRIDE: row = lane; col = 0; shP = Pt; shR = rt; break;
                        case RAP_PAT_DIAGONAL: row = lane; col = lane; shP = Pt; shR = rt; break;
                        case RAP_PAT_RANDOM: row = rrow; col = rcol; shP = Pr; shR = rr; break;
                        default:
                            row = lane; shP = Pt; shR = rt;
                            if (s == RAP_SCHEME_RAW || s == RAP_SCHEME_RAS) col = 0;
                            else if (s == RAP_SCHEME_PAD) col = (lane == 0) ? 0u : w - lane;
                            else col = lane;
                            break;
                        }
                        const uint32_t sh = (s == RAP_SCHEME_RAP) ? shP : shR;
                        uint32_t bank;
                        if (s == RAP_SCHEME_RAS || s == RAP_SCHEME_RAP) bank = mod_w<W>(col + sh, w);
                        else if (s == RAP_SCHEME_PAD) bank = mod_w<W>(row + col, w);
                        else if (s == RAP_SCHEME_XOR) bank = col ^ row;
                        else bank = col;
                        c = max_bank_load(bank, p == RAP_PAT_RANDOM ? leaders : active, ls);
                    }
                    if (p == RAP_PAT_STRIDE) c_stride[s] = c;
                    if (p == RAP_PAT_DIAGONAL) c_diag[s] = c;
                    mine = (lane == e) ? c : mine;
                    ++e;
                }
            }
            if (lane < e) atomicAdd(&sh_hist[lane * (w + 1) + mine], 1u);
        }
        __syncwarp();
    }
    __syncthreads();
    for (uint32_t b = threadIdx.x; b < nbins; b += blockDim.x)
        if (sh_hist[b]) atomicAdd((unsigned long long *)(hist + b), (unsigned long long)sh_hist[b]);
}

// ------------------------------------------------------------------ C1-C4 sweep, w = 32
// Same two phases as sweep_kernel, but for w = 32 every bank mask B_b (bit t = bit b of the bank
// of lane t) is built without per-lane arithmetic where the paper's patterns allow it:
//   * the broadcast permutation planes ARE the masks of the RAP stride access (bank = P[t]);
//   * rotations (contiguous access: bank = t + s) are funnel-shift rotations of the constant
//     lane-index masks;
//   * the diagonal access (bank = t + P[t] mod 32) is a 5-bit bit-sliced ripple-carry add;
//   * only data-dependent banks (random cells) take 5 ballots.
// The congestion is then popc / reduce-max over lane v's mask AND_b (v_b ? B_b : ~B_b) as before.
__device__ __forceinline__ uint32_t lane_bits(int b) {
    return b == 0 ? 0xAAAAAAAAu : b == 1 ? 0xCCCCCCCCu : b == 2 ? 0xF0F0F0F0u : b == 3 ? 0xFF00FF00u : 0xFFFF0000u;
}

struct BankMask { uint32_t b[5]; };

__device__ __forceinline__ BankMask masks_ballot(uint32_t bank) {   // bits 0..4 of bank (bank mod 32)
    BankMask B;
    ballot_planes5(bank, B.b);
    return B;
}

__device__ __forceinline__ BankMask masks_lane() {           // bank = t
    BankMask B;
#pragma unroll
    for (int k = 0; k < 5; ++k) B.b[k] = lane_bits(k);
    return B;
}

__device__ __forceinline__ BankMask masks_const(uint32_t v) {   // every lane the same bank v
    BankMask B;
#pragma unroll
    for (int k = 0; k < 5; ++k) B.b[k] = ((v >> k) & 1u) ? kFull : 0u;
    return B;
}

__device__ __forceinline__ BankMask masks_rot(uint32_t s) {     // bank = (t + s) mod 32
    BankMask B;
#pragma unroll
    for (int k = 0; k < 5; ++k) B.b[k] = __funnelshift_r(lane_bits(k), lane_bits(k), s);
    return B;
}

__device__ __forceinline__ BankMask masks_add(const BankMask &X, const BankMask &Y) {   // (x + y) mod 32
    BankMask S;
    uint32_t c = 0;
#pragma unroll
    for (int k = 0; k < 5; ++k) {
        S.b[k] = X.b[k] ^ Y.b[k] ^ c;
        c = (X.b[k] & Y.b[k]) | (c & (X.b[k] ^ Y.b[k]));
    }
    return S;
}

__device__ __forceinline__ uint32_t max_load(const BankMask &B, uint32_t counted, const LaneSel &ls) {
    return __reduce_max_sync(kFull, __popc(lanes_equal(B.b, counted, ls)));
}

// RAP_SWEEP_PACKED_MAX (ablation, default 0): the per-trial warp maxima reduced two at a time --
// two lane values (<= 32) packed as 16x2 halves, five SHFL.BFLY + VIMNMX.U16x2 steps -- instead of
// one CREDUX each, to unload the ADU pipe (the busiest in profiles/r02_prof_sweep.*).  Measured
// 2.99 against 3.47 G trials/s (profiles/r02_ab_sweep5.txt): the 60 extra instructions per trial
// cost more than the 8 reductions they replace.  Bit-identical; kept for the record.
#ifndef RAP_SWEEP_PACKED_MAX
#define RAP_SWEEP_PACKED_MAX 0
#endif
__device__ __forceinline__ uint32_t warp_max_16x2(uint32_t x) {
#pragma unroll
    for (int d = 16; d >= 1; d >>= 1) x = __vimax3_u16x2(x, __shfl_xor_sync(kFull, x, d), 0u);
    return x;
}

// Per-lane constants of the two rewritten evaluators below (lane v):
//   E    = AND_k (L_k ^ nsel_k)  -- bit t set iff t == v (the incidence mask of the identity map)
//   M_k  = L_k ^ nsel_k          -- bit t set iff bit k of t equals bit k of v
struct LaneEq {
    uint32_t E, M[5];
    __device__ __forceinline__ explicit LaneEq(const LaneSel &ls) {
        E = kFull;
#pragma unroll
        for (int k = 0; k < 5; ++k) {
            M[k] = lane_bits(k) ^ ls.nsel[k];
            E &= M[k];
        }
    }
};

// max_load(masks_rot(s), kFull): bank(t) = (t + s) mod 32.  Rotation commutes with AND and with
// XOR by an all-zero / all-one word, so AND_k (rotr(L_k, s) ^ nsel_k) = rotr(AND_k (L_k ^ nsel_k), s)
// = rotr(E, s): lane v's incidence mask {t : (t + s) mod 32 = v} in one funnel shift instead of
// 5 shifts + 5 LOP3 (bit-identical; tests/test_gpu_parity.py).
__device__ __forceinline__ uint32_t lane_load_rot(uint32_t s, const LaneEq &le) {
    return __popc(__funnelshift_r(le.E, le.E, s));
}
__device__ __forceinline__ uint32_t max_load_rot(uint32_t s, const LaneEq &le) {
    return __reduce_max_sync(kFull, lane_load_rot(s, le));
}

// max_load(masks_add(masks_lane(), Y), kFull): bank(t) = (t + y_t) mod 32, y_t given as planes
// Y_k.  The ripple-carry sum bit S_k = L_k ^ Y_k ^ c is produced already XORed with the lane's
// selector (S_k ^ nsel_k = Y_k ^ c ^ M_k, one LOP3 as before), so the incidence mask is a plain
// AND of five words: two LOP3 instead of five.
__device__ __forceinline__ uint32_t lane_load_add_lane(const BankMask &Y, const LaneEq &le) {
    uint32_t S[5], c = 0;
#pragma unroll
    for (int k = 0; k < 5; ++k) {
        const uint32_t L = lane_bits(k);
        S[k] = Y.b[k] ^ c ^ le.M[k];
        c = (L & Y.b[k]) | (c & (L ^ Y.b[k]));
    }
    return __popc(S[0] & S[1] & S[2] & S[3] & S[4]);
}
__device__ __forceinline__ uint32_t max_load_add_lane(const BankMask &Y, const LaneEq &le) {
    return __reduce_max_sync(kFull, lane_load_add_lane(Y, le));
}

// RAP_SWEEP_SMEM_BANKS (default 1): the accesses whose banks are data-dependent per lane -- RAS
// stride (bank r[t]), RAS diagonal (t + r[t]), and the random cells under RAW / RAS / RAP -- are
// counted with shared-memory atomics instead of ballots: each counted lane adds 1 to its bank's
// counter (a [32] array per evaluation and warp, conflict-free across distinct banks) and gets
// the previous count back; the congestion is the warp maximum of (previous + 1), i.e. the final
// count of the fullest bank.  That replaces 5 VOTE + 1 R2P (the ADU pipe, which co-limits the
// kernel with the ALU pipe) and the mask algebra by one ATOMS (the MIO / shared-memory pipe)
// per access; the counters are cleared after the trial (one STS per lane and evaluation).
#ifndef RAP_SWEEP_SMEM_BANKS
#define RAP_SWEEP_SMEM_BANKS 1
#endif
// RAP_SWEEP_DEDUP_SMEM (default 1): the merged requests of the random access (equal cells)
// are found with a 1024-bit shared-memory bitmap of the warp's cells instead of __match_any_sync:
// each lane sets its cell's bit with one atom.shared.or and leads its cell iff the bit was clear
// (lanes of one instruction to the same word are serialised, so exactly one lane per distinct cell
// finds it clear -- any one representative per cell gives the same count per bank).  MATCH.ANY's
// result latency held 29 % of the sweep's stall samples (profiles/r02_prof_sweep.source.csv.gz),
// and MATCH.ANY was what loaded the "ADU" pipe (86 % busy with it, 0.6 % without).  The bitmap is
// slot 7 of the warp's counter block and is cleared with the counters.  3.837 -> 4.571 G trials/s
// (+19 %), 4.765 with RAP_SWEEP_BATCH_HIST (profiles/r02c_ab_sweep_dedup.txt); bit-identical.
#ifndef RAP_SWEEP_DEDUP_SMEM
#define RAP_SWEEP_DEDUP_SMEM 1
#endif
constexpr int kSmemBankEvals = RAP_SWEEP_DEDUP_SMEM ? 8 : 7;   // RAS stride, RAS diagonal, random
                                                                 // under each of the 5 schemes (+ bitmap)

// RAP_SWEEP_HIST_SA (ablation, default 0): histogram increments through a shared-window address
// kept in a register instead of atomicAdd on a generic pointer (whose conversion re-reads the CTA
// window base per trial, an S2UR + ULEA carrying 17 % of the stall samples).  Measured 3.445
// against 3.466 G trials/s (profiles/r02_ab_sweep6.txt): the extra live register costs more than
// the conversion -- the stall samples only marked where the warps waited.
#ifndef RAP_SWEEP_HIST_SA
#define RAP_SWEEP_HIST_SA 0
#endif
// += 1 on a shared-memory u32 given its shared-window address
__device__ __forceinline__ void smem_inc(uint32_t saddr) {
    asm volatile("red.shared.add.u32 [%0], 1;" :: "r"(saddr) : "memory");
}

__device__ __forceinline__ uint32_t count_in_bank(uint32_t *cnt, uint32_t bank, bool counted) {
    // every lane issues the atomic (a merged duplicate adds 0 to its leader's bank): no branch
    const uint32_t one = counted ? 1u : 0u;
    return (atomicAdd(cnt + (bank & 31u), one) + 1u) * one;
}

// RAP_SWEEP_BANK4 (default 1): the sweep's data-dependent banks are carried pre-multiplied by 4
// (the byte offset of the bank's counter): the transpose buffer holds r << 12 | cell << 2, P[row]
// is assembled in bits 2..6, and a bank-counter address is one LOP3 -- (bank4 & 0x7c) | slot
// base, the slots 128-byte aligned -- instead of shift, mask and add.  Junk below bit 2 (from
// the shifts) never carries into the bank bits: every operand added to it has bits 0..1 clear.
// 8 fewer instructions per trial; +0.5 % with the STS.128 result slots (3.613 vs 3.594 G
// trials/s, profiles/r02_ab_sweep_bank4.txt), -0.3 % without them.
#ifndef RAP_SWEEP_BANK4
#define RAP_SWEEP_BANK4 1
#endif
__device__ __forceinline__ uint32_t count_in_bank4(uint32_t cnt_sa, int slot, uint32_t bank4, bool counted) {
    const uint32_t one = counted ? 1u : 0u;
    uint32_t a, old;
    // one LOP3: cnt_sa | (bank4 & 0x7c) (written out: the compiler otherwise emits AND + IADD);
    // the slot offset folds into the ATOMS address immediate
    asm("lop3.b32 %0, %1, 0x7c, %2, 0xf8;" : "=r"(a) : "r"(cnt_sa), "r"(bank4));
    asm volatile("atom.shared.add.u32 %0, [%1], %2;" : "=r"(old) : "r"(a + 128u * (uint32_t)slot), "r"(one) : "memory");
    return (old + 1u) * one;
}

// Evaluation bookkeeping of sweep32_kernel, all compile-time: evaluation e = (pattern p, scheme s)
// in mask order; "fixed" = trial-invariant (non-random pattern under RAW / PAD / XOR); "dup" =
// malicious access equal to the stride (RAW, RAS) or diagonal (RAP, XOR) access (reading iii).
__host__ __device__ constexpr int eval_index(uint32_t PM, uint32_t SM, int p, int s) {
    return __builtin_popcount(PM & ((1u << p) - 1u)) * __builtin_popcount(SM) +
           __builtin_popcount(SM & ((1u << s) - 1u));
}
__host__ __device__ constexpr bool eval_fixed(int p, int s) {
    return p != RAP_PAT_RANDOM && (s == RAP_SCHEME_RAW || s == RAP_SCHEME_PAD || s == RAP_SCHEME_XOR);
}
__host__ __device__ constexpr int eval_dup_src(uint32_t PM, uint32_t SM, int p, int s) {   // -1: not a duplicate
    return (p != RAP_PAT_MALICIOUS || eval_fixed(p, s)) ? -1
         : ((s == RAP_SCHEME_RAW || s == RAP_SCHEME_RAS) && ((PM >> RAP_PAT_STRIDE) & 1u))
               ? eval_index(PM, SM, RAP_PAT_STRIDE, s)
         : ((s == RAP_SCHEME_RAP || s == RAP_SCHEME_XOR) && ((PM >> RAP_PAT_DIAGONAL) & 1u))
               ? eval_index(PM, SM, RAP_PAT_DIAGONAL, s) : -1;
}
struct LiveEvals { int n; int idx[25]; };
__host__ __device__ constexpr LiveEvals live_evals(uint32_t PM, uint32_t SM) {      // evaluated per trial, in order
    LiveEvals L{0, {}};
    for (int p = 0; p < 5; ++p)
        for (int s = 0; s < 5; ++s)
            if (((PM >> p) & 1u) && ((SM >> s) & 1u) && !eval_fixed(p, s) && eval_dup_src(PM, SM, p, s) < 0)
                L.idx[L.n++] = eval_index(PM, SM, p, s);
    return L;
}
// position of each evaluation among the live evaluations (-1: trial-invariant or a duplicate),
// as a table built at compile time (indexed with the unrolled evaluation index)
struct LivePos { int pos[25]; };
__host__ __device__ constexpr LivePos live_pos_table(uint32_t PM, uint32_t SM) {
    LivePos T{};
    for (int e = 0; e < 25; ++e) T.pos[e] = -1;
    const LiveEvals L = live_evals(PM, SM);
    for (int i = 0; i < L.n; ++i) T.pos[L.idx[i]] = i;
    return T;
}

// RAP_SWEEP_ONEHOT (ablation, default 0): the per-trial warp maxima of all live evaluations in
// two reductions instead of one CREDUX.MAX each (9 for the cfg2 sweep), to unload the ADU pipe
// (the kernel's busiest, 78 % in profiles/r02_prof_sweep.*).  Measured 3.390 against 3.470 G
// trials/s (profiles/r02_ab_sweep_onehot.txt): with no CREDUX left on the fast path the ADU pipe
// still reads 81 % (profiles/r02_prof_sweep_onehot.raw.csv) -- its load follows the instruction
// count, not the reductions -- and the one-hot words cost 10 instructions per trial more.
// Bit-identical (every sweep parity test, profiles/r02_pytest_sweep_onehot.log).  Lane v's count c_i(v) of
// live evaluation i sets bit  min(c_i(v), width_i - 1)  of field i of a 64-bit word pair
// (u0, u1); __reduce_or_sync of each word over the warp leaves in field i exactly the set of
// counts that occur, and its highest bit is the maximum -- the congestion -- unless it is the
// field's top bit, which only says "at least width_i - 1": then (a warp-uniform branch, rare)
// the exact maxima are taken with one CREDUX.MAX per evaluation as before.  The histogram is
// therefore the same for every trial, whatever the widths.  Fields: one byte (counts 0..6 exact,
// top bit ">= 7"; a max load >= 7 has probability ~1e-3 for w = 32) per evaluation, one nibble
// (0..2, ">= 3") for the accesses a rotation or Theorem 2 makes conflict-free (contiguous under
// RAS / RAP, stride under RAP: count 1 in every trial), two nibbles per byte -- 8 bytes for the
// cfg2 sweep.  Lane e then reads its field in three operations: PRMT brings the field's byte of
// (u0, u1) to byte 3, an AND keeps the field's bits, FLO finds the highest (the count plus the
// field's bit offset 24 or 28, folded into the histogram row base).  Sets that need more than 8
// bytes keep the exact reductions.
#ifndef RAP_SWEEP_ONEHOT
#define RAP_SWEEP_ONEHOT 0
#endif
// RAP_SWEEP_PLANES_SMEM (default 1): the lane-mode phase leaves each trial's permutation planes,
// P[0] and r[0] in shared memory (two 16-byte rows per trial) and the warp-mode phase reads trial
// m's with two broadcast LDS.128 instead of seven SHFL; RAP_SWEEP_CLEAR_VEC (default 1): the bank
// counters of a trial are cleared with STS.128 spread over the lanes (2 instructions for the 5
// slots of the cfg2 sweep) instead of one STS per slot.  Both cut MIO-pipe instructions, as the
// result-slot stores below did: 3.613 -> 3.816 G trials/s together (planes +5.0 %, clears +0.5 %;
// profiles/r02_ab_sweep_planes.txt).
#ifndef RAP_SWEEP_PLANES_SMEM
#define RAP_SWEEP_PLANES_SMEM 1
#endif
#ifndef RAP_SWEEP_CLEAR_VEC
#define RAP_SWEEP_CLEAR_VEC 1
#endif
// RAP_SWEEP_RES_VEC (default 1): lane 0 stores the per-trial result slots with STS.128 (4 slots
// per instruction) instead of one predicated STS per evaluation: 3.467 -> 3.591 G trials/s
// (profiles/r02_ab_sweep_resvec.txt) -- a predicated one-lane STS still takes a full MIO slot
#ifndef RAP_SWEEP_RES_VEC
#define RAP_SWEEP_RES_VEC 1
#endif
// RAP_SWEEP_BATCH_HIST (default 1): the per-trial congestions of a batch of 32 trials are kept in
// shared memory (lane 0's STS.128 result slots, one 64-byte row per trial) and counted into the
// histogram once per batch -- lane e walks the 32 rows of its evaluation -- instead of one LDS +
// atomic (and the rematerialised shared-window address of the histogram, 19 % of the stall
// samples in profiles/r02_prof_sweep.source.csv.gz) per trial.  The room comes from the lane-mode
// transpose buffer, now 16-bit (r << 10 | cell: 15 bits, rows of 34 halves: still conflict-free);
// the buffer and the 32 result rows fit the 4224 bytes the 32-bit buffer took.  For up to 16
// evaluations (the cfg2 sweep has 15).  +4.2 % (4.571 -> 4.765 G trials/s with the bitmap dedupe,
// profiles/r02c_ab_sweep_dedup.txt).
#ifndef RAP_SWEEP_BATCH_HIST
#define RAP_SWEEP_BATCH_HIST 1
#endif
// RAP_SWEEP_PACK_SLOTS (default 1; with the batch histogram): a trial's row holds only its live
// evaluations (9 for the cfg2 sweep: no slot for the trial-invariant RAW / PAD / XOR accesses nor
// for the malicious accesses that repeat the stride / diagonal ones) -- two STS.128 and one STS
// instead of four STS.128 with zeros to fill; the lane of a duplicate reads its source's slot.
// Before the P table ptxas spent 5 more LOP3 elsewhere in the loop for it (4.672 vs 4.768 G
// trials/s, profiles/r02c_ab_sweep_mulhi.txt); with the P table the loop is 97 -> 92 instructions
// and 5.307 -> 5.452 G trials/s (profiles/r02c_ab_sweep_pack2.txt; unroll 2 5.04 / 5.45).
#ifndef RAP_SWEEP_PACK_SLOTS
#define RAP_SWEEP_PACK_SLOTS 1
#endif
// RAP_SWEEP_PBYTES (default 1, with the bitmap dedupe and the batch histogram, RAW / RAS / RAP
// schemes): the lane-mode phase turns its trial's permutation planes into a 32-byte table 4 P[t]
// (t = 0..31; nibble k of plane b spread over 4 bytes by one multiply, (nib * 0x00204081) &
// 0x01010101) in the 32-byte shared row that held the planes, so that the warp-mode phase reads
// P[t] and P[row_t] with one LDS.U8 each instead of the 14-instruction bit gather, and counts the
// RAP stride (bank P[t]) and diagonal (bank t + P[t]) accesses with the shared-memory bank
// counters (slots 5 and 6) instead of the bit-sliced mask algebra; r[0] comes from the 16-bit
// transpose buffer.  Warp-mode loop 124 -> 97 instructions, 190 -> 166 per trial in all: 4.763 ->
// 5.305 G trials/s (+11 %, profiles/r02c_ab_sweep_pbytes.txt); bit-identical.
#ifndef RAP_SWEEP_PBYTES
#define RAP_SWEEP_PBYTES 1
#endif
// RAP_SWEEP_FY_BYTES (ablation, default 0; with RAP_SWEEP_PBYTES): the lane-mode Durstenfeld
// shuffle runs directly on the lane's 32-byte P table in shared memory (a[i] = 4 i; swap a[k],
// a[j] = two LDS.U8 and two STS.U8) instead of on 5 bit planes that are converted afterwards: ~6
// instead of ~19 instructions per swap, no conversion.  The table's words are XOR-swizzled by
// (row >> 2) & 7 so that the step's common index k (the same in every lane) hits 32 distinct
// banks; the random j costs ~2-3 wavefronts.  161 -> 147 instructions per trial, but issue fell
// from 77 to 67 % (short scoreboard, MIO throttle: the swap chain's shared-memory round trips):
// 5.31 vs 5.45 G trials/s, also with the other domains' Philox interleaved into the FY loop
// (RAP_SWEEP_FY_INTERLEAVE) -- profiles/r02c_ab_sweep_fyb*.txt, r02c_prof_sweep_fyb.raw.csv.
// Bit-identical.
#ifndef RAP_SWEEP_FY_BYTES
#define RAP_SWEEP_FY_BYTES 0
#endif
#ifndef RAP_SWEEP_FY_INTERLEAVE
#define RAP_SWEEP_FY_INTERLEAVE 1
#endif
// RAP_SWEEP_UNROLL_M (tuning): unroll factor of the per-trial warp-mode loop (1: none).  Measured
// with the default 8 CTAs of 64 registers per SM: unroll 2 3.797 vs 3.839 G trials/s, and 7 / 6
// CTAs per SM with more registers 3.786 / 3.746 (profiles/r02c_ab_sweep_unroll.txt)
#ifndef RAP_SWEEP_UNROLL_M
#define RAP_SWEEP_UNROLL_M 1
#endif
constexpr int kSweepUnrollM = RAP_SWEEP_UNROLL_M;
// RAP_SWEEP_LEAD_LANE (default 1): with the bank counters every merged-request test reads only the
// lane's own leader bit, so the lane tests its own __match_any_sync word ((same & lanes below) ==
// 0) instead of gathering every lane's bit with a ballot: one VOTE fewer per trial; 3.800 -> 3.819
// G trials/s (+0.5 %, profiles/r02c_ab_sweep_pred.txt).
#ifndef RAP_SWEEP_LEAD_LANE
#define RAP_SWEEP_LEAD_LANE 1
#endif
// RAP_SWEEP_HIST_PRED (ablation, default 0): a branch-free per-trial histogram step -- the result
// slots stored by a predicated STS.128, every lane adding 0 or 1 with one red.shared -- instead of
// a branch around the 11 incrementing lanes (BSSY, BRA, two BSYNC, WARPSYNC per trial).  The loop
// loses those 5 control instructions (the ADU pipe's, 86 % busy in profiles/r02_prof_sweep.*),
// yet ran 0.3 % slower (3.788 vs 3.800 G trials/s) and ncu still shows the ADU pipe 85 % busy
// (profiles/r02c_prof_sweep_pred.raw.csv): the branch was not what loaded it.  Bit-identical.
#ifndef RAP_SWEEP_HIST_PRED
#define RAP_SWEEP_HIST_PRED 0
#endif
__device__ __forceinline__ void smem_add(uint32_t saddr, uint32_t v) {
    asm volatile("red.shared.add.u32 [%0], %1;" :: "r"(saddr), "r"(v) : "memory");
}
// 16-byte shared store executed only where `on` (a predicate in PTX, not a branch around it)
__device__ __forceinline__ void sts128_if(uint32_t saddr, uint32_t a, uint32_t b, uint32_t c, uint32_t d, bool on) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %5, 0;\n\t@p st.shared.v4.u32 [%0], {%1, %2, %3, %4};\n\t}"
                 :: "r"(saddr), "r"(a), "r"(b), "r"(c), "r"(d), "r"((uint32_t)on) : "memory");
}

__host__ __device__ constexpr bool eval_narrow(int p, int s) {
    return (p == RAP_PAT_CONTIGUOUS && (s == RAP_SCHEME_RAS || s == RAP_SCHEME_RAP)) ||
           (p == RAP_PAT_STRIDE && s == RAP_SCHEME_RAP);
}
struct OneHotLayout {
    bool fits;                                       // <= 8 bytes: two words
    int bit[kMaxEval], width[kMaxEval];              // per live evaluation i: first bit (0..63), 8 or 4
    uint32_t sat0, sat1;                             // top bits of the fields of u0 / u1
};
__host__ __device__ constexpr OneHotLayout onehot_layout(uint32_t PM, uint32_t SM) {
    OneHotLayout O{false, {}, {}, 0u, 0u};
    int nbyte = 0, half = -1, i = 0;                 // half: byte whose high nibble is free
    for (int p = 0; p < 5; ++p)
        for (int s = 0; s < 5; ++s) {
            if (!(((PM >> p) & 1u) && ((SM >> s) & 1u)) || eval_fixed(p, s) || eval_dup_src(PM, SM, p, s) >= 0)
                continue;
            if (eval_narrow(p, s)) {
                O.width[i] = 4;
                if (half >= 0) { O.bit[i] = 8 * half + 4; half = -1; }
                else { half = nbyte++; O.bit[i] = 8 * half; }
            } else {
                O.width[i] = 8;
                O.bit[i] = 8 * nbyte++;
            }
            if (nbyte <= 8) {
                const int top = O.bit[i] + O.width[i] - 1;
                if (top < 32) O.sat0 |= 1u << top; else O.sat1 |= 1u << (top - 32);
            }
            ++i;
        }
    O.fits = nbyte <= 8;
    return O;
}

template <uint32_t PM, uint32_t SM>
__global__ void __launch_bounds__(kSweepWarpsV2 * 32, RAP_SWEEP_MINB)
sweep32_kernel(uint32_t, uint32_t, uint32_t, uint64_t seed, uint64_t first, uint64_t n_trials,
               uint64_t *__restrict__ hist) {
    constexpr uint32_t w = 32;
    constexpr uint32_t npat = __builtin_popcount(PM), nsch = __builtin_popcount(SM);
    constexpr uint32_t nbins = npat * nsch * (w + 1);
    constexpr bool any_random = (PM >> RAP_PAT_RANDOM) & 1u;
    constexpr bool need_r = (SM >> RAP_SCHEME_RAS) & 1u;
    __shared__ uint32_t sh_hist[nbins];
    __shared__ __align__(16) uint32_t sh_tr[kSweepWarpsV2][32 * 33];   // 16: batch result rows take STS.128
    __shared__ __align__(16) uint32_t sh_res[kSweepWarpsV2][32];
    __shared__ __align__(128) uint32_t sh_cnt[RAP_SWEEP_SMEM_BANKS ? kSweepWarpsV2 : 1][kSmemBankEvals][32];
    __shared__ __align__(16) uint32_t sh_pl[RAP_SWEEP_PLANES_SMEM ? kSweepWarpsV2 : 1][RAP_SWEEP_PLANES_SMEM ? 32 : 1][8];
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    for (uint32_t b = threadIdx.x; b < nbins; b += blockDim.x) sh_hist[b] = 0;
    sh_res[warp][lane] = 0u;                      // slots no evaluation writes stay in range
    __syncthreads();
    const LaneSel ls(lane);
    const LaneEq le(ls);
    const uint32_t lt_mask = (1u << lane) - 1u;
    uint32_t *tr = sh_tr[warp];
    uint32_t *res = sh_res[warp];
    uint32_t *cnt = &sh_cnt[RAP_SWEEP_SMEM_BANKS ? warp : 0][0][0];
    constexpr bool kB4 = RAP_SWEEP_BANK4 && RAP_SWEEP_SMEM_BANKS && !RAP_SWEEP_PACKED_MAX && !RAP_SWEEP_ONEHOT;
    constexpr bool kDedup = RAP_SWEEP_DEDUP_SMEM && kB4 && RAP_SWEEP_LEAD_LANE && RAP_SWEEP_CLEAR_VEC;
    // batch histogram: 16-bit transpose buffer (pitch 34 halves = 17 words: row t starts in bank
    // 17 t mod 32, distinct, so the column read stays conflict-free) + 32 result rows of 16 slots
    constexpr bool kBatch = RAP_SWEEP_BATCH_HIST && kB4 && RAP_SWEEP_RES_VEC && !RAP_SWEEP_HIST_PRED &&
                            !RAP_SWEEP_HIST_SA && npat * nsch <= 16;
    uint16_t *tr16 = reinterpret_cast<uint16_t *>(sh_tr[warp]);
    uint32_t *res_b = sh_tr[warp] + 544;                 // byte 2176: after 32 x 34 u16, 16-aligned
    static_assert(!kBatch || 544 + 32 * 16 <= 32 * 33, "batch result rows fit the transpose buffer");
    constexpr bool kPB = RAP_SWEEP_PBYTES && kDedup && kBatch && RAP_SWEEP_PLANES_SMEM &&
                         !((SM >> RAP_SCHEME_PAD) & 1u) && !((SM >> RAP_SCHEME_XOR) & 1u);
    constexpr bool kFYB = kPB && RAP_SWEEP_FY_BYTES;
    constexpr bool kPack = kBatch && RAP_SWEEP_PACK_SLOTS;
    constexpr int kNLive = live_evals(PM, SM).n;
    constexpr LivePos kPos = live_pos_table(PM, SM);
    uint32_t my_slot = lane;                             // the row slot lane e reads in the batch flush
    if (kPack) {
#pragma unroll
        for (int p = 0; p < 5; ++p) {
#pragma unroll
            for (int s = 0; s < 5; ++s) {
                if (!((PM >> p) & 1u) || !((SM >> s) & 1u)) continue;
                const int e = eval_index(PM, SM, p, s), d = eval_dup_src(PM, SM, p, s);
                const int pos = kPos.pos[d >= 0 ? d : e];
                if (lane == (uint32_t)e && pos >= 0) my_slot = (uint32_t)pos;
            }
        }
    }
    const uint32_t cnt_sa = (uint32_t)__cvta_generic_to_shared(cnt);   // 128-byte aligned slots
    const uint32_t hist_sa0 = (uint32_t)__cvta_generic_to_shared(sh_hist);
    static_assert(nbins >= 32, "HIST_PRED: idle lanes add 0 to word `lane` of the histogram");
#if RAP_SWEEP_HIST_SA
    uint32_t hist_sa;                 // opaque to the compiler: kept, not rematerialised per trial
    asm volatile("mov.u32 %0, %1;" : "=r"(hist_sa) : "r"((uint32_t)__cvta_generic_to_shared(sh_hist)));
#endif
    constexpr bool kSB = RAP_SWEEP_SMEM_BANKS != 0;
    // counter slots in use: 0 RAS stride, 1 RAS diagonal (and malicious, which reuses them), 2 + s
    // the random access under scheme s
    constexpr uint32_t kSlots = (((SM >> RAP_SCHEME_RAS) & 1u) && ((PM >> RAP_PAT_STRIDE) & 1u) ? 1u : 0u) |
                                (((SM >> RAP_SCHEME_RAS) & 1u) && ((PM >> RAP_PAT_DIAGONAL) & 1u) ? 2u : 0u) |
                                (((PM >> RAP_PAT_RANDOM) & 1u) ? (SM << 2) : 0u) |
                                (RAP_SWEEP_PBYTES && RAP_SWEEP_DEDUP_SMEM && RAP_SWEEP_BATCH_HIST &&
                                 !((SM >> RAP_SCHEME_PAD) & 1u) && !((SM >> RAP_SCHEME_XOR) & 1u) &&
                                 ((SM >> RAP_SCHEME_RAP) & 1u) ? 0x60u : 0u);   // PBYTES: RAP stride 5, diagonal 6
    if (kSB) {
#pragma unroll
        for (int e = 0; e < kSmemBankEvals; ++e) cnt[e * 32 + lane] = 0u;
        __syncwarp();
    }

    // Accesses whose banks do not depend on the trial's draws -- every non-random pattern under
    // the deterministic maps RAW / PAD / XOR -- have the same congestion in every trial:
    // evaluate them once here (same evaluator) and count that value per trial below.
    uint32_t cfix[5][5];
#pragma unroll
    for (int p = 0; p < 5; ++p) {
#pragma unroll
        for (int s = 0; s < 5; ++s) {
            cfix[p][s] = 0;
            if (!((PM >> p) & 1u) || !((SM >> s) & 1u) || p == RAP_PAT_RANDOM) continue;
            if (s != RAP_SCHEME_RAW && s != RAP_SCHEME_PAD && s != RAP_SCHEME_XOR) continue;
            const int pp = (p == RAP_PAT_MALICIOUS)
                ? ((s == RAP_SCHEME_RAW) ? RAP_PAT_STRIDE : (s == RAP_SCHEME_PAD) ? -1 : RAP_PAT_DIAGONAL) : p;
            uint32_t row, col;
            switch (pp) {
            case RAP_PAT_CONTIGUOUS: row = 0; col = lane; break;
            case RAP_PAT_STRIDE: row = lane; col = 0; break;
            case RAP_PAT_DIAGONAL: row = lane; col = lane; break;
            default: row = lane; col = (32u - lane) & 31u; break;       // PAD anti-diagonal
            }
            const uint32_t bank = s == RAP_SCHEME_PAD ? ((row + col) & 31u) : s == RAP_SCHEME_XOR ? (col ^ row) : col;
            cfix[p][s] = max_load(masks_ballot(bank), kFull, ls);
        }
    }
    // evaluation slots of the trial-invariant accesses (bit e) and, for lane e, its congestion:
    // they are counted once per batch (+nvalid) instead of once per trial
    uint32_t fixed_slots = 0, fix_lane = 0;
    {
        uint32_t e = 0;
#pragma unroll
        for (int p = 0; p < 5; ++p) {
#pragma unroll
            for (int s = 0; s < 5; ++s) {
                if (!((PM >> p) & 1u) || !((SM >> s) & 1u)) continue;
                if (p != RAP_PAT_RANDOM && (s == RAP_SCHEME_RAW || s == RAP_SCHEME_PAD || s == RAP_SCHEME_XOR)) {
                    fixed_slots |= 1u << e;
                    if (lane == e) fix_lane = cfix[p][s];
                }
                ++e;
            }
        }
    }
    const bool lane_fixed = (fixed_slots >> lane) & 1u;
#if RAP_SWEEP_PACKED_MAX
    // where lane e finds its evaluation's per-trial congestion: pair slot and half (a duplicate
    // reads its source's)
    uint32_t res_slot = 0, res_shift = 0;
    {
        constexpr LiveEvals LL = live_evals(PM, SM);
#pragma unroll
        for (int p = 0; p < 5; ++p) {
#pragma unroll
            for (int s = 0; s < 5; ++s) {
                if (!((PM >> p) & 1u) || !((SM >> s) & 1u)) continue;
                const int e = eval_index(PM, SM, p, s);
                const int src = eval_dup_src(PM, SM, p, s) >= 0 ? eval_dup_src(PM, SM, p, s) : e;
#pragma unroll
                for (int i = 0; i < LL.n; ++i)
                    if (LL.idx[i] == src && lane == (uint32_t)e) {
                        res_slot = (uint32_t)(i / 2);
                        res_shift = (i & 1) ? 16u : 0u;
                    }
            }
        }
    }
#elif RAP_SWEEP_ONEHOT
    static_assert(RAP_SWEEP_SMEM_BANKS, "one-hot maxima: lane values from the bank counters");
    // lane e's evaluation (a duplicate: its source's): live index oh_i; oh_info = the PRMT
    // selector that brings its field's byte to byte 3 (bits 12..14) | the field's bits there
    // (bits 24..31, PRMT reads bits 0..15 only); oh_base = its histogram row - the FLO offset
    uint32_t oh_i = 0, oh_info = 0, oh_base = 0;
    {
        constexpr LiveEvals LL = live_evals(PM, SM);
        constexpr OneHotLayout O = onehot_layout(PM, SM);
#pragma unroll
        for (int p = 0; p < 5; ++p) {
#pragma unroll
            for (int s = 0; s < 5; ++s) {
                if (!((PM >> p) & 1u) || !((SM >> s) & 1u)) continue;
                const int e = eval_index(PM, SM, p, s);
                const int src = eval_dup_src(PM, SM, p, s) >= 0 ? eval_dup_src(PM, SM, p, s) : e;
#pragma unroll
                for (int i = 0; i < LL.n; ++i)
                    if (LL.idx[i] == src && lane == (uint32_t)e) {
                        const uint32_t nib = (uint32_t)(O.bit[i] & 7), off = 24u + nib;
                        oh_i = (uint32_t)i;
                        oh_info = ((uint32_t)(O.bit[i] >> 3) << 12) | ((((1u << O.width[i]) - 1u) << off));
                        oh_base = lane * (w + 1) - off;
                    }
            }
        }
        // opaque: kept in registers, not rematerialised per trial from the lane index
        asm volatile("mov.b32 %0, %0;" : "+r"(oh_info));
        asm volatile("mov.b32 %0, %0;" : "+r"(oh_base));
    }
#endif

    const uint64_t nbatch = (n_trials + 31) / 32;
    const uint64_t stride = (uint64_t)gridDim.x * kSweepWarpsV2;
    for (uint64_t bt = (uint64_t)blockIdx.x * kSweepWarpsV2 + warp; bt < nbatch; bt += stride) {
        const uint64_t n0 = first + bt * 32;
        const uint32_t nvalid = (uint32_t)min((uint64_t)32, n_trials - bt * 32);
        // ---- lane mode: trial n0 + lane
        uint32_t pl[5] = {0u, 0u, 0u, 0u, 0u};
        uint32_t p0_lane = 0;
        if constexpr (kFYB) {
            // C2 on the lane's byte table (row `lane` of this warp's P rows, words swizzled)
            uint8_t *rowb = reinterpret_cast<uint8_t *>(&sh_pl[warp][lane][0]);
            const uint32_t swz = ((lane >> 2) & 7u) << 2;             // byte-index XOR
#pragma unroll
            for (uint32_t q = 0; q < 8; ++q)                            // a[i] = 4 i
                reinterpret_cast<uint32_t *>(rowb)[q ^ (swz >> 2)] = 0x0C080400u + 0x10101010u * q;
#pragma unroll
            for (int blk = 0; blk < 8; ++blk) {
                const uint4 c = philox_block(seed, n0 + lane, kDomainFY, blk);
                const uint32_t u[4] = {c.x, c.y, c.z, c.w};
#if RAP_SWEEP_FY_INTERLEAVE
                // C1 of the RAS / random domains for the same block here, so that their Philox
                // arithmetic fills the latency of the swap chain's shared-memory round trips
                if (need_r || any_random) {
                    const uint4 cr = need_r ? philox_block(seed, n0 + lane, kDomainRAS, blk) : make_uint4(0, 0, 0, 0);
                    const uint4 cc = any_random ? philox_block(seed, n0 + lane, kDomainRandom, blk) : make_uint4(0, 0, 0, 0);
                    const uint32_t ur[4] = {cr.x, cr.y, cr.z, cr.w};
                    const uint32_t uc[4] = {cc.x, cc.y, cc.z, cc.w};
#pragma unroll
                    for (int i = 0; i < 4; ++i)
                        tr16[(4 * blk + i) * 34 + lane] = (uint16_t)(((ur[i] >> 27) << 10) | (uc[i] >> 22));
                }
#endif
#pragma unroll
                for (int i = 0; i < 4; ++i) {
                    const int t = 4 * blk + i;
                    if (t >= 31) break;
                    const uint32_t k = 31u - (uint32_t)t, j = mulshift(u[i], k + 1);
                    const uint8_t ak = rowb[k ^ swz], aj = rowb[j ^ swz];
                    rowb[k ^ swz] = aj;
                    rowb[j ^ swz] = ak;
                }
            }
        } else {
            lane_perm_planes<32>(seed, n0 + lane, w, pl);
            p0_lane = plane_value(pl, 0);                              // P[0] of this lane's trial
        }
        uint32_t r0_lane = 0;
        if ((need_r || any_random) && !(kFYB && RAP_SWEEP_FY_INTERLEAVE)) {
#pragma unroll
            for (int blk = 0; blk < 8; ++blk) {
                const uint4 cr = need_r ? philox_block(seed, n0 + lane, kDomainRAS, blk) : make_uint4(0, 0, 0, 0);
                const uint4 cc = any_random ? philox_block(seed, n0 + lane, kDomainRandom, blk) : make_uint4(0, 0, 0, 0);
                const uint32_t ur[4] = {cr.x, cr.y, cr.z, cr.w};
                const uint32_t uc[4] = {cc.x, cc.y, cc.z, cc.w};
#pragma unroll
                for (int i = 0; i < 4; ++i) {
                    const uint32_t r = ur[i] >> 27, cell = uc[i] >> 22;   // floor(u*32/2^32), floor(u*1024/2^32)
                    if (blk == 0 && i == 0) r0_lane = r;
                    if (kBatch) tr16[(4 * blk + i) * 34 + lane] = (uint16_t)((r << 10) | cell);
                    else tr[(4 * blk + i) * 33 + lane] = kB4 ? (r << 12) | (cell << 2) : (r << 10) | cell;
                }
            }
        }
#if RAP_SWEEP_PLANES_SMEM
        if constexpr (kFYB) {
            // (the table is already in place)
        } else if constexpr (kPB) {          // 4 P[t] as bytes: word k holds t = 4k .. 4k+3
            uint32_t pw[8];
#pragma unroll
            for (int k = 0; k < 8; ++k) {
                uint32_t x = 0;
#pragma unroll
                for (int b = 0; b < 5; ++b)
                    x |= ((((pl[b] >> (4 * k)) & 15u) * 0x00204081u) & 0x01010101u) << (b + 2);
                pw[k] = x;
            }
            *reinterpret_cast<uint4 *>(&sh_pl[warp][lane][0]) = make_uint4(pw[0], pw[1], pw[2], pw[3]);
            *reinterpret_cast<uint4 *>(&sh_pl[warp][lane][4]) = make_uint4(pw[4], pw[5], pw[6], pw[7]);
        } else {
            *reinterpret_cast<uint4 *>(&sh_pl[warp][lane][0]) = make_uint4(pl[0], pl[1], pl[2], pl[3]);
            *reinterpret_cast<uint4 *>(&sh_pl[warp][lane][4]) = make_uint4(pl[4], p0_lane, r0_lane, 0u);
        }
#endif
        __syncwarp();
        // ---- warp mode: lane t is DMM thread t of trial n0 + m
#pragma unroll kSweepUnrollM
        for (uint32_t m = 0; m < nvalid; ++m) {
            BankMask Pm;                                           // bit t = bit b of P[t]
#if RAP_SWEEP_PLANES_SMEM
            uint32_t P0, r0, Pt4 = 0;                              // Pt4 (kPB): 4 P[t]
            const uint8_t *pbytes = reinterpret_cast<const uint8_t *>(&sh_pl[warp][m][0]);
            const uint32_t mswz = kFYB ? ((m >> 2) & 7u) << 2 : 0u;  // row m's byte-index XOR
            if constexpr (kPB) {
                Pt4 = pbytes[lane ^ mswz];
                P0 = (uint32_t)pbytes[mswz] >> 2;                  // broadcast
                r0 = (uint32_t)tr16[m] >> 10;                      // r[0] of trial m (row 0)
#pragma unroll
                for (int b = 0; b < 5; ++b) Pm.b[b] = 0u;          // (unused)
            } else {
                const uint4 qa = *reinterpret_cast<const uint4 *>(&sh_pl[warp][m][0]);   // broadcast reads
                const uint4 qb = *reinterpret_cast<const uint4 *>(&sh_pl[warp][m][4]);
                Pm.b[0] = qa.x; Pm.b[1] = qa.y; Pm.b[2] = qa.z; Pm.b[3] = qa.w; Pm.b[4] = qb.x;
                P0 = qb.y; r0 = qb.z;
            }
#else
#pragma unroll
            for (int b = 0; b < 5; ++b) Pm.b[b] = __shfl_sync(kFull, pl[b], m);
            const uint32_t P0 = __shfl_sync(kFull, p0_lane, m);
            const uint32_t r0 = __shfl_sync(kFull, r0_lane, m);
#endif
            const uint32_t packed = kBatch ? (uint32_t)tr16[lane * 34 + m] << 2 : tr[lane * 33 + m];
            const uint32_t rt = packed >> 10;                      // kB4: 4 r[t] (+ junk in bits 0..1)
            BankMask Rm;
            if (need_r && !kSB) Rm = masks_ballot(rt);              // bit t = bit b of r[t]
            uint32_t rrow = 0, rcol = 0, Pr = 0, rr = 0, leaders = kFull;
            bool lead_me = true;                                   // this lane leads its cell
            if (any_random) {
                const uint32_t cell = kB4 ? packed & 0xffcu : packed & 1023u;
                rrow = kB4 ? cell >> 7 : cell >> 5;
                rcol = kB4 ? cell & 0x7cu : cell & 31u;            // kB4: 4 col
#if RAP_SWEEP_PLANES_SMEM
                if constexpr (kPB) Pr = pbytes[rrow ^ mswz];        // 4 P[row_t]
                else
#endif
                Pr = kB4 ? plane_value4(Pm.b, rrow) : plane_value(Pm.b, rrow);   // (4) P[row_t]
                rr = __shfl_sync(kFull, rt, rrow);                 // (4) r[row_t]
                if constexpr (kDedup) {                            // merged requests: cell bitmap
                    // kB4: cell = 4 x (32 row + col); the word of the cell is `row`, its bit `col`
                    const uint32_t bit = 1u << ((cell >> 2) & 31u);
                    uint32_t old;
                    asm volatile("atom.shared.or.b32 %0, [%1], %2;"
                                 : "=r"(old) : "r"(cnt_sa + 7u * 128u + ((cell >> 5) & 0x7cu)), "r"(bit) : "memory");
                    lead_me = (old & bit) == 0u;                   // the one lane that set the bit
                } else if (kSB && RAP_SWEEP_LEAD_LANE) {
                    const uint32_t same = __match_any_sync(kFull, cell);   // merged requests
                    lead_me = (same & lt_mask) == 0u;              // first lane of its cell
                } else {
                    const uint32_t same = __match_any_sync(kFull, cell);   // merged requests
                    leaders = ballot_zero(same, lt_mask);          // first lane of its cell
                    lead_me = (leaders >> lane) & 1u;
                }
            }
#if RAP_SWEEP_PACKED_MAX || RAP_SWEEP_ONEHOT
            // lane values of the evaluations done per trial, then their warp maxima (two at a
            // time, or every one of them through the one-hot words)
            constexpr int NE = npat * nsch;
            uint32_t lv[NE];
#pragma unroll
            for (int p = 0; p < 5; ++p) {
                if (!((PM >> p) & 1u)) continue;
#pragma unroll
                for (int s = 0; s < 5; ++s) {
                    if (!((SM >> s) & 1u)) continue;
                    const int e = eval_index(PM, SM, p, s);
                    lv[e] = 0u;
                    if (eval_fixed(p, s) || eval_dup_src(PM, SM, p, s) >= 0) continue;
                    const bool isp = (s == RAP_SCHEME_RAP);
                    if (kSB && ((s == RAP_SCHEME_RAS && (p == RAP_PAT_STRIDE || p == RAP_PAT_DIAGONAL ||
                                                         p == RAP_PAT_MALICIOUS)) || p == RAP_PAT_RANDOM)) {
                        // shared-memory bank counters (slot: RAS stride 0, RAS diagonal 1, random
                        // under scheme s 2 + s); the malicious RAS access is the stride access
                        const bool stride_like = p == RAP_PAT_STRIDE || p == RAP_PAT_MALICIOUS;
                        const int slot = stride_like ? 0 : p == RAP_PAT_DIAGONAL ? 1 : 2 + s;
                        const uint32_t bank = stride_like ? rt : p == RAP_PAT_DIAGONAL ? lane + rt
                                            : s == RAP_SCHEME_RAW ? packed
                                            : s == RAP_SCHEME_PAD ? rrow + rcol
                                            : s == RAP_SCHEME_XOR ? (rcol ^ rrow)
                                            : packed + (isp ? Pr : rr);
                        lv[e] = count_in_bank(cnt + slot * 32, bank, p != RAP_PAT_RANDOM || lead_me);
                    } else if (p == RAP_PAT_CONTIGUOUS) {                          // RAS / RAP
                        lv[e] = lane_load_rot(isp ? P0 : r0, le);
                    } else if (p == RAP_PAT_DIAGONAL || (p == RAP_PAT_MALICIOUS && isp)) {   // RAP (RAS: counters)
                        lv[e] = lane_load_add_lane(Pm, le);
                    } else if (p == RAP_PAT_STRIDE || p == RAP_PAT_MALICIOUS) {   // RAP stride
                        lv[e] = __popc(lanes_equal(Pm.b, kFull, ls));
                    }
                }
            }
            constexpr LiveEvals LL = live_evals(PM, SM);
#if RAP_SWEEP_PACKED_MAX
            // pair i of live evaluations -> res[i] = (max of the second) << 16 | max of the first;
            // lane e of the histogram step reads its evaluation's half (res_slot / res_shift)
#pragma unroll
            for (int i = 0; i + 1 < LL.n; i += 2) {
                const uint32_t x = warp_max_16x2(lv[LL.idx[i]] + (lv[LL.idx[i + 1]] << 16));
                if (lane == 0) res[i / 2] = x;
            }
            if (LL.n & 1) {
                const uint32_t x = __reduce_max_sync(kFull, lv[LL.idx[LL.n - 1]]);
                if (lane == 0) res[LL.n / 2] = x;
            }
#else
            // one-hot fields (RAP_SWEEP_ONEHOT): bit min(c, width - 1) of field i, OR over the warp
            constexpr OneHotLayout O = onehot_layout(PM, SM);
            uint32_t hidx;                                 // this lane's histogram bin
            uint32_t u0 = 0, u1 = 0;
            bool sat = !O.fits;
            if constexpr (O.fits) {
#pragma unroll
                for (int i = 0; i < LL.n; ++i) {
                    const uint32_t bitv = (1u << (O.bit[i] & 31)) << min(lv[LL.idx[i]], (uint32_t)(O.width[i] - 1));
                    if (O.bit[i] < 32) u0 |= bitv; else u1 |= bitv;
                }
                u0 = __reduce_or_sync(kFull, u0);
                if (O.sat1) u1 = __reduce_or_sync(kFull, u1);
                sat = ((u0 & O.sat0) | (u1 & O.sat1)) != 0u;
            }
            if (sat) {                                     // a top bit: exact maxima (warp-uniform)
#pragma unroll
                for (int i = 0; i < LL.n; ++i) {
                    const uint32_t x = __reduce_max_sync(kFull, lv[LL.idx[i]]);
                    if (lane == 0) res[i] = x;
                }
                __syncwarp();
                hidx = lane * (w + 1) + res[oh_i];
            } else {
                hidx = oh_base + (31u - __clz(__byte_perm(u0, u1, oh_info) & oh_info));
            }
#endif
            const uint32_t e = npat * nsch;
#else
            uint32_t e = 0;
            uint32_t c_stride[5] = {0, 0, 0, 0, 0}, c_diag[5] = {0, 0, 0, 0, 0};
#if RAP_SWEEP_RES_VEC
            uint32_t cres[(npat * nsch + 3) & ~3u];        // result slots, stored 4 at a time
#pragma unroll
            for (uint32_t k = (kPack ? kNLive : 0u); k < ((npat * nsch + 3) & ~3u); ++k) cres[k] = 0u;
#endif
#pragma unroll
            for (int p = 0; p < 5; ++p) {
                if (!((PM >> p) & 1u)) continue;
#pragma unroll
                for (int s = 0; s < 5; ++s) {
                    if (!((SM >> s) & 1u)) continue;
                    uint32_t c;
                    if (p != RAP_PAT_RANDOM &&
                        (s == RAP_SCHEME_RAW || s == RAP_SCHEME_PAD || s == RAP_SCHEME_XOR)) {
                        c = cfix[p][s];                             // trial-invariant access
                    } else if (p == RAP_PAT_MALICIOUS && (s == RAP_SCHEME_RAW || s == RAP_SCHEME_RAS) &&
                        ((PM >> RAP_PAT_STRIDE) & 1u)) {
                        c = c_stride[s];                            // reading iii: = stride access
                    } else if (p == RAP_PAT_MALICIOUS && (s == RAP_SCHEME_RAP || s == RAP_SCHEME_XOR) &&
                               ((PM >> RAP_PAT_DIAGONAL) & 1u)) {
                        c = c_diag[s];                              // reading iii: = diagonal access
                    } else {
                        const int pp = (p == RAP_PAT_MALICIOUS)
                            ? ((s == RAP_SCHEME_RAW || s == RAP_SCHEME_RAS) ? RAP_PAT_STRIDE
                               : (s == RAP_SCHEME_PAD) ? -1 : RAP_PAT_DIAGONAL) : p;
                        BankMask B;
                        const bool isp = (s == RAP_SCHEME_RAP);
                        const bool pb_rap = kPB && isp && (pp == RAP_PAT_STRIDE || pp == RAP_PAT_DIAGONAL);
                        if (kSB && ((s == RAP_SCHEME_RAS && (pp == RAP_PAT_STRIDE || pp == RAP_PAT_DIAGONAL)) ||
                                    pp == RAP_PAT_RANDOM || pb_rap)) {
                            // shared-memory bank counters (slot: RAS stride 0, RAS diagonal 1,
                            // random under scheme s 2 + s, PBYTES: RAP stride 5, RAP diagonal 6);
                            // packed carries rcol in bits 0..4, and count_in_bank reduces the bank
                            // mod 32
                            const int slot = pb_rap ? (pp == RAP_PAT_STRIDE ? 5 : 6)
                                           : pp == RAP_PAT_STRIDE ? 0 : pp == RAP_PAT_DIAGONAL ? 1 : 2 + s;
                            const bool counted = pp != RAP_PAT_RANDOM || lead_me;
                            if (kB4) {                             // banks as 4 x bank (counter byte offsets)
                                const uint32_t sh4 = pb_rap ? Pt4 : rt;    // 4 P[t] / 4 r[t]
                                const uint32_t bank4 = pp == RAP_PAT_STRIDE ? sh4
                                                     : pp == RAP_PAT_DIAGONAL ? (lane << 2) + sh4
                                                     : s == RAP_SCHEME_RAW ? packed
                                                     : s == RAP_SCHEME_PAD ? packed + (packed >> 5)
                                                     : s == RAP_SCHEME_XOR ? packed ^ (packed >> 5)
                                                     : packed + (isp ? Pr : rr);
                                c = __reduce_max_sync(kFull, count_in_bank4(cnt_sa, slot, bank4, counted));
                                goto counted;
                            }
                            const uint32_t bank = pp == RAP_PAT_STRIDE ? rt : pp == RAP_PAT_DIAGONAL ? lane + rt
                                                : s == RAP_SCHEME_RAW ? packed
                                                : s == RAP_SCHEME_PAD ? rrow + rcol
                                                : s == RAP_SCHEME_XOR ? (rcol ^ rrow)
                                                : packed + (isp ? Pr : rr);
                            c = __reduce_max_sync(kFull, count_in_bank(cnt + slot * 32, bank, counted));
                            goto counted;
                        }
                        if ((s == RAP_SCHEME_RAS || s == RAP_SCHEME_RAP) && pp == RAP_PAT_CONTIGUOUS) {
                            c = max_load_rot(isp ? P0 : r0, le);            // bank t + shift[0]
                            goto counted;
                        }
                        if ((s == RAP_SCHEME_RAS || s == RAP_SCHEME_RAP) && pp == RAP_PAT_DIAGONAL) {
                            c = max_load_add_lane(isp ? Pm : Rm, le);       // bank t + shift[t]
                            goto counted;
                        }
                        // (the ballots read bits 0..4 only: `packed` carries rcol in those bits,
                        // and packed + shift has (rcol + shift) mod 32 there -- the "mod w")
                        if (s == RAP_SCHEME_RAW) {
                            B = (pp == RAP_PAT_STRIDE) ? masks_const(0)
                              : (pp == RAP_PAT_RANDOM) ? masks_ballot(packed) : masks_lane();
                        } else if (s == RAP_SCHEME_RAS || s == RAP_SCHEME_RAP) {
                            if (pp == RAP_PAT_STRIDE) B = isp ? Pm : Rm;
                            else B = masks_ballot(packed + (isp ? Pr : rr));
                        } else {                                    // PAD / XOR: per-lane bank
                            uint32_t row, col;
                            switch (pp) {
                            case RAP_PAT_CONTIGUOUS: row = 0; col = lane; break;
                            case RAP_PAT_STRIDE: row = lane; col = 0; break;
                            case RAP_PAT_DIAGONAL: row = lane; col = lane; break;
                            case RAP_PAT_RANDOM: row = rrow; col = rcol; break;
                            default: row = lane; col = (32u - lane) & 31u; break;   // PAD anti-diagonal
                            }
                            B = masks_ballot(s == RAP_SCHEME_PAD ? ((row + col) & 31u) : (col ^ row));
                        }
                        c = max_load(B, pp == RAP_PAT_RANDOM ? leaders : kFull, ls);
                    }
                counted:
                    if (p == RAP_PAT_STRIDE) c_stride[s] = c;
                    if (p == RAP_PAT_DIAGONAL) c_diag[s] = c;
#if RAP_SWEEP_RES_VEC
                    if (kPack) {
                        const int pos = kPos.pos[eval_index(PM, SM, p, s)];
                        if (pos >= 0) cres[pos] = c;
                    } else if (!((fixed_slots >> e) & 1u)) {
                        cres[e] = c;
                    }
#else
                    if (lane == 0 && !((fixed_slots >> e) & 1u)) res[e] = c;   // C4: result slot e
#endif
                    ++e;
                }
            }
#if RAP_SWEEP_RES_VEC
#if RAP_SWEEP_HIST_PRED
            {                                                  // C4: the result slots, STS.128,
                const uint32_t rsa = (uint32_t)__cvta_generic_to_shared(res);   // predicated on lane 0
#pragma unroll
                for (uint32_t k = 0; k < ((npat * nsch + 3) & ~3u); k += 4)
                    sts128_if(rsa + 4u * k, cres[k], cres[k + 1], cres[k + 2], cres[k + 3], lane == 0);
            }
#else
            if (lane == 0) {                                   // C4: the result slots, STS.128
                uint32_t *rr = kBatch ? res_b + m * 16 : res;   // batch: row m of the batch
                constexpr uint32_t nst = kPack ? (uint32_t)kNLive : (npat * nsch + 3) & ~3u;
#pragma unroll
                for (uint32_t k = 0; k + 4 <= nst; k += 4)
                    *reinterpret_cast<uint4 *>(rr + k) = make_uint4(cres[k], cres[k + 1], cres[k + 2], cres[k + 3]);
#pragma unroll
                for (uint32_t k = nst & ~3u; k < nst; ++k) rr[k] = cres[k];   // the packed tail
            }
#endif
#endif
#endif
            __syncwarp();
#if RAP_SWEEP_PACKED_MAX
            if (lane < e && !lane_fixed)
                atomicAdd(&sh_hist[lane * (w + 1) + ((res[res_slot] >> res_shift) & 0xffffu)], 1u);
#elif RAP_SWEEP_ONEHOT
            if (lane < e && !lane_fixed) atomicAdd(&sh_hist[hidx], 1u);
#else
#if RAP_SWEEP_HIST_SA
            if (lane < e && !lane_fixed) smem_inc(hist_sa + 4u * (lane * (w + 1) + res[lane]));
#elif RAP_SWEEP_HIST_PRED
            // every lane adds: lane e of a live evaluation 1 to its bin, the others 0 to word `lane`
            // of the histogram (in range, distinct banks) -- no branch, no predicate to if-convert
            {
                const bool on = lane < e && !lane_fixed;
                const uint32_t bin = on ? lane * (w + 1) + res[lane] : lane;
                smem_add(hist_sa0 + 4u * bin, on ? 1u : 0u);
            }
#else
            if (!kBatch && lane < e && !lane_fixed) atomicAdd(&sh_hist[lane * (w + 1) + res[lane]], 1u);
#endif
#endif
            if (kSB) {                                                  // clear the bank counters
#if RAP_SWEEP_CLEAR_VEC
                // every slot up to the highest in use, 16 bytes per lane (unused slots stay 0)
                constexpr uint32_t kClr = (kDedup ? (kSlots | 0x80u) : kSlots);
                constexpr uint32_t n4 = kClr ? 8u * (32u - __builtin_clz(kClr)) : 0u;
#pragma unroll
                for (uint32_t i = 0; i < n4; i += 32)
                    if (i + 32 <= n4 || i + lane < n4)
                        reinterpret_cast<uint4 *>(cnt)[i + lane] = make_uint4(0u, 0u, 0u, 0u);
#else
#pragma unroll
                for (int k = 0; k < kSmemBankEvals; ++k)
                    if ((kSlots >> k) & 1u) cnt[k * 32 + lane] = 0u;
#endif
            }
            __syncwarp();
        }
        if (lane_fixed) atomicAdd(&sh_hist[lane * (w + 1) + fix_lane], nvalid);   // trial-invariant slots
        if (kBatch && lane < npat * nsch && !lane_fixed) {        // C4 of the batch: lane e, row m
            uint32_t *hrow = &sh_hist[lane * (w + 1)];
#pragma unroll 4
            for (uint32_t m = 0; m < nvalid; ++m) atomicAdd(hrow + res_b[m * 16 + my_slot], 1u);
        }
        __syncwarp();
    }
    __syncthreads();
    for (uint32_t b = threadIdx.x; b < nbins; b += blockDim.x)
        if (sh_hist[b]) atomicAdd((unsigned long long *)(hist + b), (unsigned long long)sh_hist[b]);
}

// ------------------------------------------------------------------ C1-C4 sweep (ablation)
// The north-star sketch, kept as a measured alternative: one warp per trial, Philox blocks
// spread over lanes, warp Fisher-Yates by __shfl_sync, __match_any_sync histogram.
template <int W>
__global__ void __launch_bounds__(kSweepWarps * 32)
sweep_match_kernel(uint32_t w_rt, uint32_t pmask, uint32_t smask, uint64_t seed, uint64_t first,
                   uint64_t n_trials, uint64_t *__restrict__ hist) {
    const uint32_t w = W ? (uint32_t)W : w_rt;
    __shared__ uint32_t sh_hist[kSweepWarps][kMaxBins];
    __shared__ __align__(16) uint32_t sh_words[kSweepWarps][4 * 32];
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    const uint32_t npat = __popc(pmask), nsch = __popc(smask);
    const uint32_t nbins = npat * nsch * (w + 1);
    for (uint32_t b = lane; b < nbins; b += 32) sh_hist[warp][b] = 0;
    __syncwarp();

    const bool any_random = (pmask >> RAP_PAT_RANDOM) & 1u;
    const uint64_t stride = (uint64_t)gridDim.x * kSweepWarps;
    for (uint64_t i = (uint64_t)blockIdx.x * kSweepWarps + warp; i < n_trials; i += stride) {
        const uint64_t n = first + i;
        const uint4 blk = philox_block(seed, n, lane >> 3, lane & 7u);
        *reinterpret_cast<uint4 *>(&sh_words[warp][4 * lane]) = blk;   // word(d,t) at [32d + t]
        __syncwarp();
        const uint32_t u_fy = sh_words[warp][lane];
        const uint32_t u_ras = sh_words[warp][32 + lane];
        const uint32_t u_rnd = sh_words[warp][64 + lane];
        __syncwarp();
        const uint32_t P = warp_fisher_yates<W>(u_fy, lane, w);
        const uint32_t r = mulshift(u_ras, w);
        uint32_t rrow = 0, rcol = 0;
        if (any_random) {
            const uint32_t cell = mulshift(u_rnd, w * w);
            if (W == 32) { rrow = cell >> 5; rcol = cell & 31u; }
            else { rrow = cell / w; rcol = cell - rrow * w; }
        }
        uint32_t mine = 0, e = 0;
#pragma unroll
        for (int p = 0; p < 5; ++p) {
            if (!((pmask >> p) & 1u)) continue;
#pragma unroll
            for (int s = 0; s < 5; ++s) {
                if (!((smask >> s) & 1u)) continue;
                uint32_t row, col;
                pattern_cell(p, s, lane, w, rrow, rcol, row, col);
                const uint32_t c = warp_congestion_match<W>(row, col, s, P, r, lane, w, p == RAP_PAT_RANDOM);
                mine = (lane == e) ? c : mine;
                ++e;
            }
        }
        if (lane < e) sh_hist[warp][lane * (w + 1) + mine] += 1;
    }
    flush_hist(sh_hist, kSweepWarps, nbins, hist);
}

// ------------------------------------------------------------------ trace evaluator
constexpr int kTraceChunk = 32;

// RAP_TRACE_MINB: CTAs per SM the register budget is cut for (4: 64 registers, 32 warps per SM)
#ifndef RAP_TRACE_MINB
#define RAP_TRACE_MINB 4
#endif
// W: compile-time w (32: the default bank count, cells split by shift / mask), 0: runtime w.
// SM: compile-time scheme mask (0: runtime).  The merge of identical addresses depends only on
// the cells, so the leaders (one lane per distinct cell, one __match_any_sync) are found once per
// trace warp and shared by the schemes; each scheme then costs one shuffle (its shift of the
// request's row), the bank map and the ballot histogram.
template <int W, uint32_t SM>
__global__ void __launch_bounds__(kSweepWarps * 32, RAP_TRACE_MINB)
trace_kernel(uint32_t w_rt, uint64_t n_warps, const uint32_t *__restrict__ cells, uint32_t smask_rt,
             uint64_t seed, uint64_t first, uint64_t n_trials, uint64_t *__restrict__ hist) {
    const uint32_t w = W ? (uint32_t)W : w_rt;
    const uint32_t smask = SM ? SM : smask_rt;
    __shared__ uint32_t sh_hist[kSweepWarps][kMaxBins];
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    const uint32_t nsch = __popc(smask);
    const uint32_t nbins = nsch * (w + 1);
    for (uint32_t b = lane; b < nbins; b += 32) sh_hist[warp][b] = 0;
    __syncwarp();
    const LaneSel ls(lane);
    const uint32_t active = (w >= 32) ? kFull : ((1u << w) - 1u);
    const uint32_t lt_mask = (1u << lane) - 1u;
    const bool need_p = (smask >> RAP_SCHEME_RAP) & 1u, need_r = (smask >> RAP_SCHEME_RAS) & 1u;
    const uint64_t nchunks = (n_warps + kTraceChunk - 1) / kTraceChunk;
    const uint64_t nitems = n_trials * nchunks;
    const uint64_t stride = (uint64_t)gridDim.x * kSweepWarps;
    for (uint64_t it = (uint64_t)blockIdx.x * kSweepWarps + warp; it < nitems; it += stride) {
        const uint64_t trial = it / nchunks, chunk = it - trial * nchunks;
        const uint64_t n = first + trial;
        const uint32_t P = need_p ? warp_perm<W>(seed, n, lane, w) : lane;
        const uint32_t r = need_r ? warp_ras_shift(seed, n, lane, w) : 0u;
        const uint64_t k_end = min(n_warps, (chunk + 1) * kTraceChunk);
        uint32_t next = (lane < w) ? __ldg(cells + chunk * kTraceChunk * w + lane) : 0u;
        for (uint64_t k = chunk * kTraceChunk; k < k_end; ++k) {
            const uint32_t raw_cell = next;                            // the next trace warp's
            if (k + 1 < k_end) next = (lane < w) ? __ldg(cells + (k + 1) * w + lane) : 0u;   // load in flight
            const bool bad = __any_sync(kFull, raw_cell >= w * w);   // counted in bin 0
            const uint32_t cell = bad ? 0u : raw_cell;
            const uint32_t row = (W == 32) ? (cell >> 5) : cell / w;
            const uint32_t col = (W == 32) ? (cell & 31u) : cell - row * w;
            // merged requests: the first lane of each distinct cell is counted
            const uint32_t same = __match_any_sync(kFull, (lane < w) ? cell : (0x40000000u | lane));
            const uint32_t leaders = ballot_zero(same, lt_mask) & active;
            uint32_t mine = 0, e = 0;
#pragma unroll
            for (int s = 0; s < 5; ++s) {
                if (!((smask >> s) & 1u)) continue;
                uint32_t bank;
                if (s == RAP_SCHEME_RAS || s == RAP_SCHEME_RAP)
                    bank = mod_w<W>(col + __shfl_sync(kFull, s == RAP_SCHEME_RAP ? P : r, row & 31u), w);
                else if (s == RAP_SCHEME_PAD) bank = mod_w<W>(row + col, w);
                else if (s == RAP_SCHEME_XOR) bank = col ^ row;
                else bank = col;
                const uint32_t c = max_bank_load(bank, leaders, ls);
                mine = (lane == e) ? (bad ? 0u : c) : mine;
                ++e;
            }
            if (lane < e) sh_hist[warp][lane * (w + 1) + mine] += 1;
        }
    }
    flush_hist(sh_hist, kSweepWarps, nbins, hist);
}


// w = 32 trace evaluator.  Work unit = (block of kTraceTB trials, range of kTraceTK trace warps).
// The CTA first draws P and r of its kTraceTB trials into shared memory (one warp Fisher-Yates
// per trial), then each warp takes trace warps of the range and, per trace warp:
//   * decodes the 32 cells and finds the merged-request leaders ONCE (one __match_any_sync);
//   * evaluates the trial-invariant schemes RAW / PAD / XOR once and counts the result for every
//     trial of the block (their bank maps use no random numbers);
//   * for each trial of the block evaluates RAS / RAP: the shift of the lane's row is one LDS.U8
//     (P_t[row] -- lanes of equal rows share a word, so one wavefront), bank = col + shift (the
//     ballots read bits 0..4 only, which is the "mod 32"), 5 ballots, popc, reduce-max.
// Histograms live in registers: lane L of the warp counts congestion L+1 for each scheme, flushed
// with one u64 atomic per non-zero counter at the end.
#ifndef RAP_TRACE_GENERIC
#define RAP_TRACE_GENERIC 0
#endif
#ifndef RAP_TRACE_TB
#define RAP_TRACE_TB 32
#endif
// trace warps per unit: the per-trial P / r draws of a unit are shared by its TK trace warps.
// Measured with the BANK4 counters (4096 trace warps x 2048 trials): TK 64 105.1, 128 111.9,
// 192 112.3, 256 105.4 G warp-evaluations/s (fewer units than 2 waves), TB 16 x TK 128 101.2
// (profiles/r02c_ab_trace*.txt)
#ifndef RAP_TRACE_TK
#define RAP_TRACE_TK 128
#endif
#ifndef RAP_TRACE_WARPS
#define RAP_TRACE_WARPS 8
#endif
constexpr int kTraceTB = RAP_TRACE_TB;     // trials per unit (P, r of the block in shared memory)
constexpr int kTraceTK = RAP_TRACE_TK;     // trace warps per unit
constexpr int kTraceWarps = RAP_TRACE_WARPS;

#ifndef RAP_TRACE32_MINB
#define RAP_TRACE32_MINB 4
#endif

// trace32_kernel helpers: lanes that play DMM threads, and (x mod w) for x < 2w -- for W = 32 the
// ballots read bits 0..4 only, which is already the reduction mod 32
template <int W>
__device__ __forceinline__ bool lane_active(uint32_t w) { return W == 32 || (threadIdx.x & 31u) < w; }
template <int W>
__device__ __forceinline__ uint32_t wrap_w(uint32_t x, uint32_t w) { return W == 32 ? x : (x >= w ? x - w : x); }

#ifndef RAP_TRACE_SMEM_BANKS
#define RAP_TRACE_SMEM_BANKS 1
#endif
// RAP_TRACE_BANK4 (default 1): as RAP_SWEEP_BANK4 -- the shifts are kept as 4 x shift (a byte:
// <= 124) and the lane's column as 4 x col, so a counter address is (4 col + 4 shift) & 0x7c
// OR'ed into the counter set's 128-byte-aligned base: one LOP3 instead of mask, shift and add
#ifndef RAP_TRACE_BANK4
#define RAP_TRACE_BANK4 1
#endif
// RAP_TRACE_HIST_SMEM (ablation, default 0; with RAP_TRACE_BANK4): per trial of the RAS / RAP
// loop, lane t keeps trial t's congestion (one select) instead of every lane testing c == lane + 1
// and counting (compare, add, select); after the block's trials each lane adds its value to a
// per-warp shared-memory histogram with one atomic.  59 -> 56 instructions per 4 unrolled trials,
// no measurable gain (111.73 vs 111.79 G warp-evaluations/s, profiles/r02c_ab_trace3*.txt).
#ifndef RAP_TRACE_HIST_SMEM
#define RAP_TRACE_HIST_SMEM 0
#endif
// W = 32: compile-time w (cells split by shift / mask, the ballots' bits 0..4 are the "mod 32");
// W = 0: runtime w < 32 (lanes >= w idle, explicit mod w, w + 1 bins per scheme).
template <int W, uint32_t SM>
__global__ void __launch_bounds__(kTraceWarps * 32, RAP_TRACE32_MINB)
trace32_kernel(uint32_t w_rt, uint64_t n_warps, const uint32_t *__restrict__ cells, uint64_t seed, uint64_t first,
               uint64_t n_trials, uint64_t *__restrict__ hist) {
    const uint32_t w = W ? (uint32_t)W : w_rt;
    const bool active = lane_active<W>(w);
    const uint32_t amask = (w >= 32) ? kFull : ((1u << w) - 1u);
    constexpr uint32_t nsch = __builtin_popcount(SM);
    constexpr bool need_p = (SM >> RAP_SCHEME_RAP) & 1u, need_r = (SM >> RAP_SCHEME_RAS) & 1u;
    __shared__ uint8_t shP[kTraceTB][32], shR[kTraceTB][32];
    // RAP_TRACE_SMEM_BANKS: per-trial RAS / RAP evaluations count the lanes of each bank with
    // shared-memory atomics (see RAP_SWEEP_SMEM_BANKS) -- four counter sets per warp, one per
    // trial of the unrolled loop, cleared after use
    __shared__ __align__(128) uint32_t sh_tcnt[RAP_TRACE_SMEM_BANKS ? kTraceWarps : 1][4][32];
    constexpr bool kTB4 = RAP_TRACE_BANK4 && RAP_TRACE_SMEM_BANKS && W == 32;
    constexpr bool kTHS = kTB4 && RAP_TRACE_HIST_SMEM;
    __shared__ uint32_t sh_th[kTHS ? kTraceWarps : 1][kTHS ? nsch : 1][33];   // RAS / RAP bins per warp
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    const LaneSel ls(lane);
    const uint32_t lt_mask = (1u << lane) - 1u;
    uint32_t hc[nsch];                                      // lane L: count of congestion L + 1
#pragma unroll
    for (uint32_t e = 0; e < nsch; ++e) hc[e] = 0;
    uint32_t hbad = 0;                                      // evaluations of warps with a bad cell
    if (RAP_TRACE_SMEM_BANKS && W == 32) {
#pragma unroll
        for (int k = 0; k < 4; ++k) sh_tcnt[RAP_TRACE_SMEM_BANKS ? warp : 0][k][lane] = 0u;
        __syncwarp();
    }
    if constexpr (kTHS) {
        for (uint32_t i = lane; i < nsch * 33; i += 32) (&sh_th[warp][0][0])[i] = 0u;
        __syncwarp();
    }
    const uint64_t nkc = (n_warps + kTraceTK - 1) / kTraceTK;
    const uint64_t ntb = (n_trials + kTraceTB - 1) / kTraceTB;
    for (uint64_t unit = blockIdx.x; unit < ntb * nkc; unit += gridDim.x) {
        const uint64_t tb = unit / nkc, kc = unit - tb * nkc;
        const uint64_t t0 = tb * kTraceTB;
        const uint32_t tcnt = (uint32_t)min((uint64_t)kTraceTB, n_trials - t0);
        __syncthreads();                                    // the previous unit is done with shP / shR
        for (uint32_t t = warp; t < tcnt; t += kTraceWarps) {
            if (need_p) shP[t][lane] = (uint8_t)(warp_perm<W>(seed, first + t0 + t, lane, w) << (kTB4 ? 2 : 0));
            if (need_r) shR[t][lane] = (uint8_t)(warp_ras_shift(seed, first + t0 + t, lane, w) << (kTB4 ? 2 : 0));
        }
        __syncthreads();
        const uint64_t k_end = min(n_warps, (kc + 1) * kTraceTK);
        for (uint64_t k = kc * kTraceTK + warp; k < k_end; k += kTraceWarps) {
            const uint32_t raw_cell = active ? __ldg(cells + k * w + lane) : 0u;
            if (__any_sync(kFull, active && raw_cell >= w * w)) {     // invalid trace warp: bin 0
                hbad += tcnt;
                continue;
            }
            const uint32_t row = W == 32 ? raw_cell >> 5 : raw_cell / w;
            const uint32_t col = W == 32 ? raw_cell & 31u : raw_cell - row * w;
            // merged requests: the first lane of each distinct cell is counted
            const uint32_t same = __match_any_sync(kFull, active ? raw_cell : (0x80000000u | lane));
            const uint32_t leaders = ballot_zero(same, lt_mask) & amask;
            uint32_t e = 0;
#pragma unroll
            for (int s = 0; s < 5; ++s) {
                if (!((SM >> s) & 1u)) continue;
                if (s == RAP_SCHEME_RAW || s == RAP_SCHEME_PAD || s == RAP_SCHEME_XOR) {
                    const uint32_t bank = s == RAP_SCHEME_RAW ? col : s == RAP_SCHEME_PAD ? wrap_w<W>(row + col, w) : (col ^ row);
                    const uint32_t c = max_bank_load(bank, leaders, ls);
                    hc[e] += (c == lane + 1u) ? tcnt : 0u;
                } else if (RAP_TRACE_SMEM_BANKS && W == 32) {
                    const uint8_t *sh = s == RAP_SCHEME_RAP ? &shP[0][0] : &shR[0][0];
                    uint32_t *cnt = &sh_tcnt[RAP_TRACE_SMEM_BANKS ? warp : 0][0][0];
                    const bool lead = (leaders >> lane) & 1u;
                    if constexpr (kTB4) {
                        const uint32_t cnt_sa = (uint32_t)__cvta_generic_to_shared(cnt), col4 = col << 2;
                        uint32_t mine = 0;                     // kTHS: trial `lane`'s congestion
#pragma unroll 4
                        for (uint32_t t = 0; t < tcnt; ++t) {
                            const uint32_t c = __reduce_max_sync(
                                kFull, count_in_bank4(cnt_sa, (int)(t & 3u), col4 + sh[t * 32 + row], lead));
                            __syncwarp();
                            cnt[(t & 3u) * 32 + lane] = 0u;   // every lane's increment has returned
                            if (kTHS) mine = (lane == t) ? c : mine;
                            else hc[e] += (c == lane + 1u) ? 1u : 0u;
                        }
                        if (kTHS && lane < tcnt) atomicAdd(&sh_th[kTHS ? warp : 0][kTHS ? e : 0][mine], 1u);
                    } else {
#pragma unroll 4
                    for (uint32_t t = 0; t < tcnt; ++t) {
                        uint32_t *ct = cnt + (t & 3u) * 32;
                        const uint32_t c = __reduce_max_sync(kFull, count_in_bank(ct, col + sh[t * 32 + row], lead));
                        __syncwarp();
                        ct[lane] = 0u;                     // every lane's increment has returned
                        hc[e] += (c == lane + 1u) ? 1u : 0u;
                    }
                    }
                    __syncwarp();
                } else {
                    const uint8_t *sh = s == RAP_SCHEME_RAP ? &shP[0][0] : &shR[0][0];
#pragma unroll 4
                    for (uint32_t t = 0; t < tcnt; ++t) {
                        const uint32_t c = max_bank_load(wrap_w<W>(col + sh[t * 32 + row], w), leaders, ls);
                        hc[e] += (c == lane + 1u) ? 1u : 0u;
                    }
                }
                ++e;
            }
        }
    }
    if (kTHS) __syncwarp();
#pragma unroll
    for (uint32_t e = 0; e < nsch; ++e) {
        const uint32_t v = hc[e] + (kTHS ? sh_th[kTHS ? warp : 0][kTHS ? e : 0][lane + 1] : 0u);
        if (v) atomicAdd((unsigned long long *)(hist + e * (w + 1) + lane + 1), (unsigned long long)v);
        if (lane == 0 && hbad) atomicAdd((unsigned long long *)(hist + e * (w + 1)), (unsigned long long)hbad);
    }
}

// ------------------------------------------------------------------ batched evaluator
__global__ void __launch_bounds__(256)
congestion_kernel(uint32_t w, uint64_t n_warps, const uint32_t *__restrict__ rows,
                  const uint32_t *__restrict__ cols, int scheme, const uint32_t *__restrict__ shift,
                  uint32_t *__restrict__ out) {
    const uint32_t lane = threadIdx.x & 31u;
    const LaneSel ls(lane);
    const uint64_t stride = (uint64_t)gridDim.x * (blockDim.x >> 5);
    for (uint64_t k = (uint64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); k < n_warps;
         k += stride) {
        const bool active = lane < w;
        const uint32_t row = active ? rows[k * w + lane] : 0u;
        const uint32_t col = active ? cols[k * w + lane] : 0u;
        const uint32_t sh = (active && shift) ? shift[k * w + lane] : 0u;
        const bool bad = active && (row >= w || col >= w || sh >= w);
        const bool any_bad = __any_sync(kFull, bad);
        const uint32_t c = warp_congestion(any_bad ? 0u : row, any_bad ? 0u : col, scheme,
                                           any_bad ? 0u : sh, any_bad ? 0u : sh, lane, w, ls);
        if (lane == 0) out[k] = any_bad ? 0u : c;
    }
}

// ------------------------------------------------------------------ T0 perm_gen
__global__ void __launch_bounds__(256)
perm_gen_kernel(uint64_t seed, uint64_t first, uint64_t count, uint32_t w, uint8_t *__restrict__ out) {
    const uint32_t lane = threadIdx.x & 31u;
    const uint64_t stride = (uint64_t)gridDim.x * (blockDim.x >> 5);
    for (uint64_t k = (uint64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); k < count;
         k += stride) {
        const uint32_t P = warp_perm<0>(seed, first + k, lane, w);
        if (lane < w) out[k * w + lane] = (uint8_t)P;
    }
}

// ------------------------------------------------------------------ launchers
static int sm_count() {
    static std::atomic<int> cache[kMaxDevices];
    int dev = 0, sms = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= kMaxDevices) return 148;
    sms = cache[dev].load(std::memory_order_relaxed);
    if (sms == 0) {
        if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || sms <= 0) sms = 148;
        cache[dev].store(sms, std::memory_order_relaxed);
    }
    return sms;
}

// resident CTAs of `kernel` per device (occupancy query cached per kernel and device)
template <auto Kernel>
static int resident_ctas(int threads) {
    static std::atomic<int> cache[kMaxDevices];
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= kMaxDevices) dev = 0;
    int occ = cache[dev].load(std::memory_order_relaxed);
    if (occ == 0) {
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, Kernel, threads, 0) != cudaSuccess || occ < 1) occ = 1;
        cache[dev].store(occ, std::memory_order_relaxed);
    }
    return occ * sm_count();
}

static int clamp_grid(uint64_t items, int per_cta, int cap) {
    const uint64_t want = (items + per_cta - 1) / per_cta;
    return (int)(want < (uint64_t)cap ? (want ? want : 1) : (uint64_t)cap);
}

template <auto Kernel>
static void run_sweep(int warps_per_cta, uint64_t trials_per_item, uint32_t w, uint32_t pmask,
                      uint32_t smask, uint64_t seed, uint64_t first, uint64_t n_trials, uint64_t *hist,
                      cudaStream_t st) {
    const int threads = warps_per_cta * 32;
    const uint64_t items = (n_trials + trials_per_item - 1) / trials_per_item;
    const int grid = clamp_grid(items, warps_per_cta, RAP_SWEEP_GRID_MULT * resident_ctas<Kernel>(threads));
    // u32 shared counters: keep the trials counted by one CTA below 2^31 per launch
    const uint64_t chunk = (uint64_t)grid * (1ull << 31);
    for (uint64_t done = 0; done < n_trials; done += chunk) {
        const uint64_t cnt = (n_trials - done < chunk) ? n_trials - done : chunk;
        Kernel<<<grid, threads, 0, st>>>(w, pmask, smask, seed, first + done, cnt, hist);
    }
}

cudaError_t launch_sweep(uint32_t w, uint32_t pmask, uint32_t smask, uint64_t seed, uint64_t first,
                         uint64_t n_trials, uint64_t *hist, cudaStream_t st) {
    if (n_trials == 0) return cudaSuccess;
    if (w == 32 && pmask == 31u && smask == 7u)
        run_sweep<sweep32_kernel<31u, 7u>>(kSweepWarpsV2, 32, w, pmask, smask, seed, first, n_trials, hist, st);
    else if (w == 32 && pmask == 31u && smask == 31u)
        run_sweep<sweep32_kernel<31u, 31u>>(kSweepWarpsV2, 32, w, pmask, smask, seed, first, n_trials, hist, st);
    else if (w == 32)
        run_sweep<sweep_kernel<32, 0u, 0u>>(kSweepWarpsV2, 32, w, pmask, smask, seed, first, n_trials, hist, st);
    else if (pmask == 31u && smask == 7u)      // w < 32 with the Table II masks fixed at compile time
        run_sweep<sweep_kernel<0, 31u, 7u>>(kSweepWarpsV2, 32, w, pmask, smask, seed, first, n_trials, hist, st);
    else
        run_sweep<sweep_kernel<0, 0u, 0u>>(kSweepWarpsV2, 32, w, pmask, smask, seed, first, n_trials, hist, st);
    return cudaGetLastError();
}

cudaError_t launch_sweep_match(uint32_t w, uint32_t pmask, uint32_t smask, uint64_t seed, uint64_t first,
                               uint64_t n_trials, uint64_t *hist, cudaStream_t st) {
    if (n_trials == 0) return cudaSuccess;
    if (w == 32) run_sweep<sweep_match_kernel<32>>(kSweepWarps, 1, w, pmask, smask, seed, first, n_trials, hist, st);
    else run_sweep<sweep_match_kernel<0>>(kSweepWarps, 1, w, pmask, smask, seed, first, n_trials, hist, st);
    return cudaGetLastError();
}

template <int W, uint32_t SM>
static void run_trace32(uint32_t w, uint64_t n_warps, const uint32_t *cells, uint64_t seed, uint64_t first,
                        uint64_t n_trials, uint64_t *hist, cudaStream_t st) {
    const int threads = kTraceWarps * 32;
    const uint64_t nkc = (n_warps + kTraceTK - 1) / kTraceTK;
    const int cap = resident_ctas<trace32_kernel<W, SM>>(threads);
    // per-lane u32 counters: a warp evaluates at most ceil(units / grid) units of
    // (kTraceTK / kTraceWarps) trace warps x kTraceTB trials per launch -- keep that below 2^31
    const uint64_t per_unit = (uint64_t)(kTraceTK / kTraceWarps) * kTraceTB;
    const uint64_t max_units = (1ull << 31) / per_unit;     // per CTA per launch
    const uint64_t tb_chunk = max_units * (uint64_t)cap / nkc + 1;  // trial blocks per launch
    const uint64_t trials_chunk = tb_chunk * kTraceTB;
    for (uint64_t done = 0; done < n_trials; done += trials_chunk) {
        const uint64_t cnt = (n_trials - done < trials_chunk) ? n_trials - done : trials_chunk;
        const uint64_t units = ((cnt + kTraceTB - 1) / kTraceTB) * nkc;
        const int grid = (int)(units < (uint64_t)cap ? units : (uint64_t)cap);
        trace32_kernel<W, SM><<<grid, threads, 0, st>>>(w, n_warps, cells, seed, first + done, cnt, hist);
    }
}

cudaError_t launch_trace(uint32_t w, uint64_t n_warps, const uint32_t *cells, uint32_t smask,
                         uint64_t seed, uint64_t first, uint64_t n_trials, uint64_t *hist,
                         cudaStream_t st) {
    if (n_trials == 0 || n_warps == 0) return cudaSuccess;
#if !RAP_TRACE_GENERIC
    {
#define RAPK_TRACE32(M) case M: if (w == 32) run_trace32<32, M>(w, n_warps, cells, seed, first, n_trials, hist, st); \
                                else run_trace32<0, M>(w, n_warps, cells, seed, first, n_trials, hist, st); break;
        switch (smask) {
            RAPK_TRACE32(1) RAPK_TRACE32(2) RAPK_TRACE32(3) RAPK_TRACE32(4) RAPK_TRACE32(5) RAPK_TRACE32(6)
            RAPK_TRACE32(7) RAPK_TRACE32(8) RAPK_TRACE32(9) RAPK_TRACE32(10) RAPK_TRACE32(11) RAPK_TRACE32(12)
            RAPK_TRACE32(13) RAPK_TRACE32(14) RAPK_TRACE32(15) RAPK_TRACE32(16) RAPK_TRACE32(17) RAPK_TRACE32(18)
            RAPK_TRACE32(19) RAPK_TRACE32(20) RAPK_TRACE32(21) RAPK_TRACE32(22) RAPK_TRACE32(23) RAPK_TRACE32(24)
            RAPK_TRACE32(25) RAPK_TRACE32(26) RAPK_TRACE32(27) RAPK_TRACE32(28) RAPK_TRACE32(29) RAPK_TRACE32(30)
            RAPK_TRACE32(31)
            default: return cudaErrorInvalidValue;
        }
#undef RAPK_TRACE32
        return cudaGetLastError();
    }
#endif
    // RAP_TRACE_GENERIC (ablation): the first evaluator, one warp per (trial, chunk of 32 trace
    // warps), leaders and trial-invariant schemes recomputed for every trial
    const int threads = kSweepWarps * 32;
    const uint64_t nchunks = (n_warps + kTraceChunk - 1) / kTraceChunk;
    auto kern = trace_kernel<0, 0u>;
    const int occ = resident_ctas<trace_kernel<0, 0u>>(threads);
    const int grid = clamp_grid(n_trials * nchunks, kSweepWarps, occ);
    // counts per warp <= items_per_warp * kTraceChunk; chunk the trial range to stay < 2^31
    const uint64_t trials_chunk = ((uint64_t)grid * kSweepWarps * ((1ull << 31) / kTraceChunk)) / nchunks + 1;
    for (uint64_t done = 0; done < n_trials; done += trials_chunk) {
        const uint64_t cnt = (n_trials - done < trials_chunk) ? n_trials - done : trials_chunk;
        kern<<<grid, threads, 0, st>>>(w, n_warps, cells, smask, seed, first + done, cnt, hist);
    }
    return cudaGetLastError();
}

cudaError_t launch_congestion(uint32_t w, uint64_t n_warps, const uint32_t *rows, const uint32_t *cols,
                              int scheme, const uint32_t *shift, uint32_t *out, cudaStream_t st) {
    if (n_warps == 0) return cudaSuccess;
    const int grid = clamp_grid(n_warps, 8, resident_ctas<congestion_kernel>(256));
    congestion_kernel<<<grid, 256, 0, st>>>(w, n_warps, rows, cols, scheme, shift, out);
    return cudaGetLastError();
}

cudaError_t launch_perm_gen(uint64_t seed, uint64_t first, uint64_t count, uint32_t w, uint8_t *out,
                            cudaStream_t st) {
    if (count == 0) return cudaSuccess;
    const int grid = clamp_grid(count, 8, resident_ctas<perm_gen_kernel>(256));
    perm_gen_kernel<<<grid, 256, 0, st>>>(seed, first, count, w, out);
    return cudaGetLastError();
}

}  // namespace rapk
