// sweep_wide.cu -- NEXT-3: the congestion sweep for DMMs wider than a CUDA warp, 32 < w <= 256
// (Table II's w = 64, 128, 256 columns, §V; "the value of w may be increased in
// future GPUs").
//
// Default design (sweep_wide_lane_kernel): a CUDA warp takes a batch of 32 trials.
// In LANE mode each lane runs the Durstenfeld chain of its own trial on a swizzled [k][32] byte
// table (conflict-free both for a lane-mode row and a warp-mode column read); in WARP mode lane L
// plays DMM threads L + 32i of one trial at a time -- Philox words drawn by all lanes, merged
// requests by __match_any_sync per 32-request slice plus a w^2-bit bitmap across slices, bank
// counts by shared atomics (the congestion is the largest returned count).
//
// The first design, ONE CUDA THREAD PER TRIAL (sweep_wide_kernel below, built with
// -DRAP_SWEEP_WIDE_THREAD): the thread draws its permutation (Durstenfeld on a private array),
// its RAS shifts and its random cells from the same counter contract as every other kernel
// (rap_rng.cuh / include/rap.h), then walks the w requests of each (pattern, scheme), counting
// distinct requests per bank in a private array laid out [index][thread] in shared memory.
#include <cuda_runtime.h>
#include <stdint.h>

#include "rap_rng.cuh"
#include "rap_internal.h"

namespace rapk {

constexpr int kWideThreads = 64;

// word(seed, n, d, t) for sequential t, one Philox block per 4 words
struct WordStream {
    uint64_t seed, n;
    uint32_t d, blk = 0xffffffffu;
    uint4 cur;
    __device__ uint32_t operator()(uint32_t t) {
        if ((t >> 2) != blk) {
            blk = t >> 2;
            cur = philox_block(seed, n, d, blk);
        }
        return pick(cur, t & 3u);
    }
};

__global__ void __launch_bounds__(kWideThreads)
sweep_wide_kernel(uint32_t w, uint32_t pmask, uint32_t smask, uint64_t seed, uint64_t first,
                  uint64_t n_trials, uint64_t *__restrict__ hist) {
    extern __shared__ __align__(16) uint32_t dyn[];
    const uint32_t npat = __popc(pmask), nsch = __popc(smask);
    const uint32_t nbins = npat * nsch * (w + 1);
    uint32_t *sh_hist = dyn;                                       // [nbins] CTA histogram
    uint16_t *base = reinterpret_cast<uint16_t *>(dyn + ((nbins + 3) & ~3u));
    const uint32_t T = kWideThreads, tid = threadIdx.x;
    uint16_t *a = base + tid;                                      // perm        a[k*T]
    uint16_t *r = base + (size_t)w * T + tid;                      // RAS shifts  r[k*T]
    uint16_t *cell = base + (size_t)2 * w * T + tid;               // cells       cell[t*T]
    uint16_t *cnt = base + (size_t)3 * w * T + tid;                // per-bank counters
    uint32_t *lead = reinterpret_cast<uint32_t *>(base + (size_t)4 * w * T) + tid;   // leader bits [w/32][T]
    for (uint32_t b = tid; b < nbins; b += T) sh_hist[b] = 0;
    __syncthreads();
    const bool any_random = (pmask >> RAP_PAT_RANDOM) & 1u;
    const bool need_r = (smask >> RAP_SCHEME_RAS) & 1u;

    for (uint64_t i = (uint64_t)blockIdx.x * T + tid; i < n_trials; i += (uint64_t)gridDim.x * T) {
        const uint64_t n = first + i;
        // C1 + C2: P = perm(seed, n, w), Durstenfeld (include/rap.h counter contract)
        for (uint32_t k = 0; k < w; ++k) a[k * T] = (uint16_t)k;
        WordStream fy{seed, n, kDomainFY};
        for (uint32_t k = w - 1; k >= 1; --k) {
            const uint32_t j = mulshift(fy(w - 1 - k), k + 1);
            const uint16_t x = a[k * T];
            a[k * T] = a[j * T];
            a[j * T] = x;
        }
        if (need_r) {
            WordStream rs{seed, n, kDomainRAS};
            for (uint32_t k = 0; k < w; ++k) r[k * T] = (uint16_t)mulshift(rs(k), w);
        }
        if (any_random) {
            WordStream cs{seed, n, kDomainRandom};
            for (uint32_t t = 0; t < w; ++t) cell[t * T] = (uint16_t)mulshift(cs(t), w * w);
            // merged requests: request t counts only if no earlier request has its cell
            for (uint32_t q = 0; q < (w + 31) / 32; ++q) {
                uint32_t bits = 0;
                for (uint32_t t = 32 * q; t < min(w, 32 * q + 32); ++t) {
                    const uint16_t c = cell[t * T];
                    bool first_occ = true;
                    for (uint32_t s = 0; s < t; ++s) first_occ &= (cell[s * T] != c);
                    bits |= (first_occ ? 1u : 0u) << (t - 32 * q);
                }
                lead[q * T] = bits;
            }
        }
        // C3 + C4: every selected (pattern, scheme)
        uint32_t e = 0;
        for (int p = 0; p < 5; ++p) {
            if (!((pmask >> p) & 1u)) continue;
            for (int s = 0; s < 5; ++s) {
                if (!((smask >> s) & 1u)) continue;
                int pp = p;                                        // reading iii: malicious
                if (p == RAP_PAT_MALICIOUS)
                    pp = (s == RAP_SCHEME_RAW || s == RAP_SCHEME_RAS) ? RAP_PAT_STRIDE
                       : (s == RAP_SCHEME_PAD) ? -1 : RAP_PAT_DIAGONAL;
                for (uint32_t b = 0; b < w; ++b) cnt[b * T] = 0;
                uint32_t mx = 0;
                for (uint32_t t = 0; t < w; ++t) {
                    uint32_t row, col;
                    switch (pp) {
                    case RAP_PAT_CONTIGUOUS: row = 0; col = t; break;
                    case RAP_PAT_STRIDE: row = t; col = 0; break;
                    case RAP_PAT_DIAGONAL: row = t; col = t; break;
                    case RAP_PAT_RANDOM: {
                        if (!((lead[(t >> 5) * T] >> (t & 31u)) & 1u)) continue;   // merged
                        const uint32_t c = cell[t * T];
                        row = c / w;
                        col = c - row * w;
                        break;
                    }
                    default: row = t; col = t == 0 ? 0u : w - t; break;          // PAD anti-diagonal
                    }
                    uint32_t bank;
                    if (s == RAP_SCHEME_RAS || s == RAP_SCHEME_RAP) {
                        bank = col + (s == RAP_SCHEME_RAP ? a[row * T] : r[row * T]);
                        bank = bank >= w ? bank - w : bank;
                    } else if (s == RAP_SCHEME_PAD) {
                        bank = row + col;
                        bank = bank >= w ? bank - w : bank;
                    } else if (s == RAP_SCHEME_XOR) {
                        bank = col ^ row;
                    } else {
                        bank = col;
                    }
                    const uint32_t v = cnt[bank * T] + 1u;
                    cnt[bank * T] = (uint16_t)v;
                    mx = v > mx ? v : mx;
                }
                atomicAdd(&sh_hist[e * (w + 1) + mx], 1u);
                ++e;
            }
        }
    }
    __syncthreads();
    for (uint32_t b = tid; b < nbins; b += T)
        if (sh_hist[b]) atomicAdd((unsigned long long *)(hist + b), (unsigned long long)sh_hist[b]);
}

// ---------------------------------------------------------------- one CUDA warp per trial
// The default for 32 < w <= 256.  A warp simulates one DMM warp of w threads: lane L plays DMM
// threads t = L + 32 i (i < NI = ceil(w / 32)).  Per trial, in the warp's shared-memory slice:
//   * Philox words are drawn in parallel (lane L: blocks L, L + 32 of each domain); the FY draws
//     become j_t = floor(u_t (w - t) / 2^32) in jv[], the RAS shifts r[], the random cells stay in
//     registers;
//   * Durstenfeld on a[] is one sequential chain (lane 0; k = w-1 .. 1: swap a[k], a[jv[w-1-k]]);
//   * merged requests: slice by slice, a request leads iff its atom.shared.or is the
//     one that sets its cell's bit in a w*w-bit bitmap (RAP_WIDE_DEDUP_ATOM; formerly the lowest
//     lane of its cell in the slice by __match_any_sync, bit not yet set by an earlier slice);
//     the bits are cleared again afterwards (O(w) per trial);
//   * each (pattern, scheme): every lane adds its requests to the per-bank counters cnt[] with
//     shared atomics -- congestion = max over requests of the returned count + 1 (= max over
//     banks), reduce-max over the warp -- then zeroes the counters it touched.
constexpr int kWideWarps = 8;
// RAP_WIDE_DEDUP_ATOM (default 1): a request leads iff its atom.shared.or sets the cell's bit in
// the w*w-bit bitmap (lanes of one instruction to one word are serialised: one leader per distinct
// cell, across and within slices) -- no __match_any_sync, whose latency dominated the w = 32
// sweep (DESIGN §6 C, step 4)
#ifndef RAP_WIDE_DEDUP_ATOM
#define RAP_WIDE_DEDUP_ATOM 1
#endif
#ifndef RAP_WIDE_LANE_FY
#define RAP_WIDE_LANE_FY 1
#endif
#ifndef RAP_WIDE_MINB
#define RAP_WIDE_MINB 4
#endif

struct WideSlice {           // per-warp shared-memory slice, in 32-bit words
    uint32_t *a, *r, *jv, *cnt, *bm;
};

__host__ __device__ inline uint32_t wide_warp_words(uint32_t w) {
    return 4 * w + (w * w + 31) / 32;
}

template <int NI, uint32_t PM, uint32_t SM>
__global__ void __launch_bounds__(kWideWarps * 32, RAP_WIDE_MINB)
sweep_wide_warp_kernel(uint32_t w, uint32_t pmask_rt, uint32_t smask_rt, uint64_t seed, uint64_t first,
                       uint64_t n_trials, uint64_t *__restrict__ hist) {
    const uint32_t pmask = PM ? PM : pmask_rt, smask = SM ? SM : smask_rt;
    extern __shared__ __align__(16) uint32_t dyn[];
    const uint32_t npat = __popc(pmask), nsch = __popc(smask);
    const uint32_t nbins = npat * nsch * (w + 1);
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    uint32_t *sh_hist = dyn;
    uint32_t *mine = dyn + ((nbins + 3) & ~3u) + warp * wide_warp_words(w);
    WideSlice S{mine, mine + w, mine + 2 * w, mine + 3 * w, mine + 4 * w};
    for (uint32_t b = threadIdx.x; b < nbins; b += blockDim.x) sh_hist[b] = 0;
    for (uint32_t b = lane; b < 4 * w + (w * w + 31) / 32; b += 32) mine[b] = 0;
    __syncthreads();
    const bool any_random = (pmask >> RAP_PAT_RANDOM) & 1u;
    const bool need_r = (smask >> RAP_SCHEME_RAS) & 1u;
    const uint32_t nblk = (w + 3) / 4;                      // Philox blocks per domain

    const uint64_t stride = (uint64_t)gridDim.x * kWideWarps;
    for (uint64_t i = (uint64_t)blockIdx.x * kWideWarps + warp; i < n_trials; i += stride) {
        const uint64_t n = first + i;
        // ---- C1: draws, lanes in parallel
        uint32_t cellv[NI];
#pragma unroll
        for (int q = 0; q < NI; ++q) cellv[q] = 0;
        for (uint32_t blk = lane; blk < nblk; blk += 32) {
            const uint4 f = philox_block(seed, n, kDomainFY, blk);
            const uint32_t fw[4] = {f.x, f.y, f.z, f.w};
#pragma unroll
            for (int c = 0; c < 4; ++c) {
                const uint32_t t = 4 * blk + c;               // FY word t -> k = w - 1 - t
                if (t + 1 < w) S.jv[t] = mulshift(fw[c], w - t);
            }
            if (need_r) {
                const uint4 g = philox_block(seed, n, kDomainRAS, blk);
                const uint32_t gw[4] = {g.x, g.y, g.z, g.w};
#pragma unroll
                for (int c = 0; c < 4; ++c)
                    if (4 * blk + c < w) S.r[4 * blk + c] = mulshift(gw[c], w);
            }
        }
        if (any_random) {
#pragma unroll
            for (int q = 0; q < NI; ++q) {
                const uint32_t t = lane + 32u * q;
                if (t < w) cellv[q] = mulshift(pick(philox_block(seed, n, kDomainRandom, t >> 2), t & 3u), w * w);
            }
        }
#pragma unroll
        for (int q = 0; q < NI; ++q) {
            const uint32_t t = lane + 32u * q;
            if (t < w) S.a[t] = t;
        }
        __syncwarp();
        // ---- C2: Durstenfeld, one sequential chain
        if (lane == 0) {
            const uint32_t *jp = S.jv;
            uint32_t *ak = S.a + (w - 1);
#pragma unroll 4
            for (uint32_t k = w - 1; k >= 1; --k, ++jp, --ak) {
                const uint32_t j = *jp;
                const uint32_t x = *ak;
                *ak = S.a[j];
                S.a[j] = x;
            }
        }
        // ---- merged requests of the random pattern; row / col of each random cell
        uint32_t lead = 0;                                    // bit q: request lane + 32q counts
        uint32_t rrow[NI], rcol[NI];
#pragma unroll
        for (int q = 0; q < NI; ++q) {
            rrow[q] = cellv[q] / w;
            rcol[q] = cellv[q] - rrow[q] * w;
        }
        if (any_random) {
#pragma unroll
            for (int q = 0; q < NI; ++q) {
                const uint32_t t = lane + 32u * q;
                const bool valid = t < w;
                const uint32_t c = cellv[q];
#if RAP_WIDE_DEDUP_ATOM
                if (valid) {                                  // the one lane that sets the bit leads
                    const uint32_t bit = 1u << (c & 31u);
                    if (!(atomicOr(&S.bm[c >> 5], bit) & bit)) lead |= 1u << q;
                }
                __syncwarp();
#else
                const uint32_t same = __match_any_sync(kFull, valid ? c : (0x80000000u | lane));
                const bool first_in_slice = (__ffs(same) - 1) == (int)lane;
                const bool seen = valid && ((S.bm[c >> 5] >> (c & 31u)) & 1u);
                if (valid && first_in_slice && !seen) lead |= 1u << q;
                __syncwarp();
                if (valid) atomicOr(&S.bm[c >> 5], 1u << (c & 31u));
                __syncwarp();
#endif
            }
#pragma unroll
            for (int q = 0; q < NI; ++q)
                if (lane + 32u * q < w) S.bm[cellv[q] >> 5] = 0u;
        }
        __syncwarp();
        // ---- C3 + C4: every selected (pattern, scheme)
        uint32_t e = 0;
#pragma unroll
        for (int p = 0; p < 5; ++p) {
            if (!((pmask >> p) & 1u)) continue;
#pragma unroll
            for (int s = 0; s < 5; ++s) {
                if (!((smask >> s) & 1u)) continue;
                int pp = p;                                   // reading iii: malicious
                if (p == RAP_PAT_MALICIOUS)
                    pp = (s == RAP_SCHEME_RAW || s == RAP_SCHEME_RAS) ? RAP_PAT_STRIDE
                       : (s == RAP_SCHEME_PAD) ? -1 : RAP_PAT_DIAGONAL;
                uint32_t bankv[NI];
                uint32_t mx = 0;
#pragma unroll
                for (int q = 0; q < NI; ++q) {
                    const uint32_t t = lane + 32u * q;
                    bankv[q] = 0xffffffffu;
                    if (t >= w) continue;
                    if (pp == RAP_PAT_RANDOM && !((lead >> q) & 1u)) continue;      // merged
                    uint32_t row, col;
                    switch (pp) {
                    case RAP_PAT_CONTIGUOUS: row = 0; col = t; break;
                    case RAP_PAT_STRIDE: row = t; col = 0; break;
                    case RAP_PAT_DIAGONAL: row = t; col = t; break;
                    case RAP_PAT_RANDOM: row = rrow[q]; col = rcol[q]; break;
                    default: row = t; col = t == 0 ? 0u : w - t; break;               // PAD anti-diagonal
                    }
                    uint32_t bank;
                    if (s == RAP_SCHEME_RAS || s == RAP_SCHEME_RAP) {
                        bank = col + (s == RAP_SCHEME_RAP ? S.a[row] : S.r[row]);
                        bank = bank >= w ? bank - w : bank;
                    } else if (s == RAP_SCHEME_PAD) {
                        bank = row + col;
                        bank = bank >= w ? bank - w : bank;
                    } else if (s == RAP_SCHEME_XOR) {
                        bank = col ^ row;
                    } else {
                        bank = col;
                    }
                    bankv[q] = bank;
                    const uint32_t v = atomicAdd(&S.cnt[bank], 1u) + 1u;
                    mx = v > mx ? v : mx;
                }
                mx = __reduce_max_sync(kFull, mx);
                __syncwarp();
#pragma unroll
                for (int q = 0; q < NI; ++q)
                    if (bankv[q] != 0xffffffffu) S.cnt[bankv[q]] = 0u;
                if (lane == 0) atomicAdd(&sh_hist[e * (w + 1) + mx], 1u);
                __syncwarp();
                ++e;
            }
        }
    }
    __syncthreads();
    for (uint32_t b = threadIdx.x; b < nbins; b += blockDim.x)
        if (sh_hist[b]) atomicAdd((unsigned long long *)(hist + b), (unsigned long long)sh_hist[b]);
}


// Lane-mode Durstenfeld variant (RAP_WIDE_LANE_FY, default): a warp takes a batch of 32 trials;
// in lane mode lane L runs the whole Durstenfeld chain of trial n0 + L on its own column of a
// [k][32] byte table (w <= 256 fits u8), so 32 chains advance together instead of one; then in
// warp mode the trials are evaluated one after the other as in sweep_wide_warp_kernel, the RAP
// shift of row r of trial m being byte r*32 + (m ^ sw(r)).  The XOR swizzle
// sw(k) = ((k >> 2) & 7) << 2 keeps both access shapes conflict-free: a lane-mode row k is 32
// consecutive bytes, and a warp-mode column read of 32 distinct rows lands in 32 distinct banks
// (bank = 8 (r & 3) + ((m >> 2) ^ ((r >> 2) & 7))).
__host__ __device__ inline uint32_t wide_lane_words(uint32_t w) {
    return 8 * w + 3 * w + (w * w + 31) / 32;      // perm table, r, cells, cnt, merge bitmap
}

__device__ __forceinline__ uint32_t pt_off(uint32_t k, uint32_t col) { return k * 32u + (col ^ (((k >> 2) & 7u) << 2)); }

template <int NI, uint32_t PM, uint32_t SM>
__global__ void __launch_bounds__(kWideWarps * 32, RAP_WIDE_MINB)
sweep_wide_lane_kernel(uint32_t w, uint32_t pmask_rt, uint32_t smask_rt, uint64_t seed, uint64_t first,
                       uint64_t n_trials, uint64_t *__restrict__ hist) {
    const uint32_t pmask = PM ? PM : pmask_rt, smask = SM ? SM : smask_rt;
    extern __shared__ __align__(16) uint32_t dyn[];
    const uint32_t npat = __popc(pmask), nsch = __popc(smask);
    const uint32_t nbins = npat * nsch * (w + 1);
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    uint32_t *sh_hist = dyn;
    uint32_t *mine = dyn + ((nbins + 3) & ~3u) + warp * wide_lane_words(w);
    uint8_t *pt = reinterpret_cast<uint8_t *>(mine);          // [w][32] bytes, swizzled
    uint32_t *rsh = mine + 8 * w, *cw = mine + 9 * w, *cnt = mine + 10 * w, *bm = mine + 11 * w;
    for (uint32_t b = threadIdx.x; b < nbins; b += blockDim.x) sh_hist[b] = 0;
    for (uint32_t b = lane; b < wide_lane_words(w); b += 32) mine[b] = 0;
    __syncthreads();
    const bool any_random = (pmask >> RAP_PAT_RANDOM) & 1u;
    const bool need_r = (smask >> RAP_SCHEME_RAS) & 1u;
    const uint32_t nblk = (w + 3) / 4;

    const uint64_t nbatch = (n_trials + 31) / 32;
    const uint64_t stride = (uint64_t)gridDim.x * kWideWarps;
    for (uint64_t bt = (uint64_t)blockIdx.x * kWideWarps + warp; bt < nbatch; bt += stride) {
        const uint64_t n0 = first + bt * 32;
        const uint32_t nvalid = (uint32_t)min((uint64_t)32, n_trials - bt * 32);
        // ---- C1 + C2 in lane mode: P of trial n0 + lane (include/rap.h counter contract)
        for (uint32_t k = 0; k < w; ++k) pt[pt_off(k, lane)] = (uint8_t)k;
        {
            WordStream fy{seed, n0 + lane, kDomainFY};
            for (uint32_t k = w - 1; k >= 1; --k) {
                const uint32_t j = mulshift(fy(w - 1 - k), k + 1);
                const uint32_t ok = pt_off(k, lane), oj = pt_off(j, lane);
                const uint8_t x = pt[ok];
                pt[ok] = pt[oj];
                pt[oj] = x;
            }
        }
        __syncwarp();
        // ---- warp mode: trial n0 + m
        for (uint32_t m = 0; m < nvalid; ++m) {
            const uint64_t n = n0 + m;
            for (uint32_t blk = lane; blk < nblk; blk += 32) {
                if (need_r) {
                    const uint4 g = philox_block(seed, n, kDomainRAS, blk);
                    const uint32_t gw[4] = {g.x, g.y, g.z, g.w};
#pragma unroll
                    for (int c = 0; c < 4; ++c)
                        if (4 * blk + c < w) rsh[4 * blk + c] = mulshift(gw[c], w);
                }
                if (any_random) {
                    const uint4 g = philox_block(seed, n, kDomainRandom, blk);
                    const uint32_t gw[4] = {g.x, g.y, g.z, g.w};
#pragma unroll
                    for (int c = 0; c < 4; ++c)
                        if (4 * blk + c < w) cw[4 * blk + c] = mulshift(gw[c], w * w);
                }
            }
            __syncwarp();
            uint32_t cellv[NI], rrow[NI], rcol[NI];
            uint32_t lead = 0;
            if (any_random) {
#pragma unroll
                for (int q = 0; q < NI; ++q) {
                    const uint32_t t = lane + 32u * q;
                    cellv[q] = t < w ? cw[t] : 0u;
                    rrow[q] = cellv[q] / w;
                    rcol[q] = cellv[q] - rrow[q] * w;
                }
#pragma unroll
                for (int q = 0; q < NI; ++q) {          // merged requests, slice by slice
                    const uint32_t t = lane + 32u * q;
                    const bool valid = t < w;
                    const uint32_t c = cellv[q];
#if RAP_WIDE_DEDUP_ATOM
                    if (valid) {                              // the one lane that sets the bit leads
                        const uint32_t bit = 1u << (c & 31u);
                        if (!(atomicOr(&bm[c >> 5], bit) & bit)) lead |= 1u << q;
                    }
                    __syncwarp();
#else
                    const uint32_t same = __match_any_sync(kFull, valid ? c : (0x80000000u | lane));
                    const bool first_in_slice = (__ffs(same) - 1) == (int)lane;
                    const bool seen = valid && ((bm[c >> 5] >> (c & 31u)) & 1u);
                    if (valid && first_in_slice && !seen) lead |= 1u << q;
                    __syncwarp();
                    if (valid) atomicOr(&bm[c >> 5], 1u << (c & 31u));
                    __syncwarp();
#endif
                }
#pragma unroll
                for (int q = 0; q < NI; ++q)
                    if (lane + 32u * q < w) bm[cellv[q] >> 5] = 0u;
            }
            __syncwarp();
            uint32_t e = 0;
#pragma unroll
            for (int p = 0; p < 5; ++p) {
                if (!((pmask >> p) & 1u)) continue;
#pragma unroll
                for (int s = 0; s < 5; ++s) {
                    if (!((smask >> s) & 1u)) continue;
                    int pp = p;                                   // reading iii: malicious
                    if (p == RAP_PAT_MALICIOUS)
                        pp = (s == RAP_SCHEME_RAW || s == RAP_SCHEME_RAS) ? RAP_PAT_STRIDE
                           : (s == RAP_SCHEME_PAD) ? -1 : RAP_PAT_DIAGONAL;
                    uint32_t bankv[NI];
                    uint32_t mx = 0;
#pragma unroll
                    for (int q = 0; q < NI; ++q) {
                        const uint32_t t = lane + 32u * q;
                        bankv[q] = 0xffffffffu;
                        if (t >= w) continue;
                        if (pp == RAP_PAT_RANDOM && !((lead >> q) & 1u)) continue;      // merged
                        uint32_t row, col;
                        switch (pp) {
                        case RAP_PAT_CONTIGUOUS: row = 0; col = t; break;
                        case RAP_PAT_STRIDE: row = t; col = 0; break;
                        case RAP_PAT_DIAGONAL: row = t; col = t; break;
                        case RAP_PAT_RANDOM: row = rrow[q]; col = rcol[q]; break;
                        default: row = t; col = t == 0 ? 0u : w - t; break;           // PAD anti-diagonal
                        }
                        uint32_t bank;
                        if (s == RAP_SCHEME_RAS || s == RAP_SCHEME_RAP) {
                            bank = col + (s == RAP_SCHEME_RAP ? (uint32_t)pt[pt_off(row, m)] : rsh[row]);
                            bank = bank >= w ? bank - w : bank;
                        } else if (s == RAP_SCHEME_PAD) {
                            bank = row + col;
                            bank = bank >= w ? bank - w : bank;
                        } else if (s == RAP_SCHEME_XOR) {
                            bank = col ^ row;
                        } else {
                            bank = col;
                        }
                        bankv[q] = bank;
                        const uint32_t v = atomicAdd(&cnt[bank], 1u) + 1u;
                        mx = v > mx ? v : mx;
                    }
                    mx = __reduce_max_sync(kFull, mx);
                    __syncwarp();
#pragma unroll
                    for (int q = 0; q < NI; ++q)
                        if (bankv[q] != 0xffffffffu) cnt[bankv[q]] = 0u;
                    if (lane == 0) atomicAdd(&sh_hist[e * (w + 1) + mx], 1u);
                    __syncwarp();
                    ++e;
                }
            }
        }
        __syncwarp();
    }
    __syncthreads();
    for (uint32_t b = threadIdx.x; b < nbins; b += blockDim.x)
        if (sh_hist[b]) atomicAdd((unsigned long long *)(hist + b), (unsigned long long)sh_hist[b]);
}

size_t wide_smem_bytes(uint32_t w, uint32_t pmask, uint32_t smask) {
    const uint32_t nbins = __builtin_popcount(pmask) * __builtin_popcount(smask) * (w + 1);
    return 4 * (size_t)((nbins + 3) & ~3u) + 2 * (size_t)4 * w * kWideThreads +
           4 * (size_t)((w + 31) / 32) * kWideThreads;
}

static cudaError_t launch_sweep_wide_thread(uint32_t w, uint32_t pmask, uint32_t smask, uint64_t seed,
                                            uint64_t first, uint64_t n_trials, uint64_t *hist, cudaStream_t st) {
    const size_t smem = wide_smem_bytes(w, pmask, smask);
    cudaError_t e = cudaFuncSetAttribute(sweep_wide_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    int dev = 0, sms = 148, occ = 1;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, sweep_wide_kernel, kWideThreads, smem);
    if (occ < 1) occ = 1;
    const uint64_t want = (n_trials + kWideThreads - 1) / kWideThreads;
    const uint64_t cap = (uint64_t)sms * occ;
    const int grid = (int)(want < cap ? want : cap);
    // u32 CTA counters: keep the trials of one CTA below 2^31 per launch
    const uint64_t chunk = (uint64_t)grid * (1ull << 31);
    for (uint64_t done = 0; done < n_trials; done += chunk) {
        const uint64_t cnt = (n_trials - done < chunk) ? n_trials - done : chunk;
        sweep_wide_kernel<<<grid, kWideThreads, smem, st>>>(w, pmask, smask, seed, first + done, cnt, hist);
    }
    return cudaGetLastError();
}

template <int NI>
static cudaError_t launch_wide_warp(uint32_t w, uint32_t pmask, uint32_t smask, uint64_t seed, uint64_t first,
                                    uint64_t n_trials, uint64_t *hist, cudaStream_t st) {
    const uint32_t nbins = __builtin_popcount(pmask) * __builtin_popcount(smask) * (w + 1);
    const size_t smem = 4 * ((size_t)((nbins + 3) & ~3u) + (size_t)kWideWarps * wide_warp_words(w));
    // compile-time masks for the Table II sweeps (5 patterns x RAW/RAS/RAP, and all 5 schemes)
#if RAP_WIDE_LANE_FY
    const size_t smem_l = 4 * ((size_t)((nbins + 3) & ~3u) + (size_t)kWideWarps * wide_lane_words(w));
    if (smem_l <= 227 * 1024) {
        auto kl = (pmask == 31u && smask == 7u) ? sweep_wide_lane_kernel<NI, 31u, 7u>
                : (pmask == 31u && smask == 31u) ? sweep_wide_lane_kernel<NI, 31u, 31u>
                : sweep_wide_lane_kernel<NI, 0u, 0u>;
        cudaError_t e = cudaFuncSetAttribute(kl, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_l);
        if (e != cudaSuccess) return e;
        int dev = 0, sms = 148, occ = 1;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kl, kWideWarps * 32, smem_l);
        if (occ < 1) occ = 1;
        const uint64_t want = (n_trials + 32 * kWideWarps - 1) / (32 * kWideWarps);
        const uint64_t cap = (uint64_t)sms * occ;
        const int grid = (int)(want < cap ? want : cap);
        const uint64_t chunk = (uint64_t)grid * (1ull << 31);  // u32 CTA counters stay below 2^31
        for (uint64_t done = 0; done < n_trials; done += chunk) {
            const uint64_t cnt = (n_trials - done < chunk) ? n_trials - done : chunk;
            kl<<<grid, kWideWarps * 32, smem_l, st>>>(w, pmask, smask, seed, first + done, cnt, hist);
        }
        return cudaGetLastError();
    }
#endif
    auto k = (pmask == 31u && smask == 7u) ? sweep_wide_warp_kernel<NI, 31u, 7u>
           : (pmask == 31u && smask == 31u) ? sweep_wide_warp_kernel<NI, 31u, 31u>
           : sweep_wide_warp_kernel<NI, 0u, 0u>;
    cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    int dev = 0, sms = 148, occ = 1;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k, kWideWarps * 32, smem);
    if (occ < 1) occ = 1;
    const uint64_t want = (n_trials + kWideWarps - 1) / kWideWarps;
    const uint64_t cap = (uint64_t)sms * occ;
    const int grid = (int)(want < cap ? want : cap);
    const uint64_t chunk = (uint64_t)grid * (1ull << 31);    // u32 CTA counters stay below 2^31
    for (uint64_t done = 0; done < n_trials; done += chunk) {
        const uint64_t cnt = (n_trials - done < chunk) ? n_trials - done : chunk;
        k<<<grid, kWideWarps * 32, smem, st>>>(w, pmask, smask, seed, first + done, cnt, hist);
    }
    return cudaGetLastError();
}

// RAP_SWEEP_WIDE_THREAD: the one-trial-per-thread kernel above (the round-1 design, an ablation)
cudaError_t launch_sweep_wide(uint32_t w, uint32_t pmask, uint32_t smask, uint64_t seed, uint64_t first,
                              uint64_t n_trials, uint64_t *hist, cudaStream_t st) {
    if (n_trials == 0) return cudaSuccess;
#ifdef RAP_SWEEP_WIDE_THREAD
    return launch_sweep_wide_thread(w, pmask, smask, seed, first, n_trials, hist, st);
#else
    switch ((w + 31) / 32) {
    case 2: return launch_wide_warp<2>(w, pmask, smask, seed, first, n_trials, hist, st);
    case 3: return launch_wide_warp<3>(w, pmask, smask, seed, first, n_trials, hist, st);
    case 4: return launch_wide_warp<4>(w, pmask, smask, seed, first, n_trials, hist, st);
    case 5: return launch_wide_warp<5>(w, pmask, smask, seed, first, n_trials, hist, st);
    case 6: return launch_wide_warp<6>(w, pmask, smask, seed, first, n_trials, hist, st);
    case 7: return launch_wide_warp<7>(w, pmask, smask, seed, first, n_trials, hist, st);
    case 8: return launch_wide_warp<8>(w, pmask, smask, seed, first, n_trials, hist, st);
    default: return launch_sweep_wide_thread(w, pmask, smask, seed, first, n_trials, hist, st);
    }
#endif
}

}  // namespace rapk
