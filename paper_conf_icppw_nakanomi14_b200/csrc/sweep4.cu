// sweep4.cu -- NEXT-3 part 2: the RAP for higher dimension (§VII, Table IV).
//
// A w x w x w x w array a[i][j][k][l] sits at address i*w^3 + j*w^2 + k*w + l, bank l
// (P:L1598-1602).  A scheme stores a[i][j][k][l] at a[i][j][k][(l + f(i,j,k)) mod w] with
//   RAW f = 0;   RAS f = r[i][j][k] (w^3 independent shifts, drawn on demand from domain 1 at
//   index (i*w + j)*w + k);   1P f = P[k];   R1P f = P[i] + P[j] + P[k];   3P f = P[i] + Q[j] + R[k]
// (P, Q, R: Durstenfeld permutations from domains 0, 3, 4).  One CUDA warp = one DMM warp
// (w <= 32); lane t requests contiguous (0,0,0,t), stride1 (0,0,t,0), stride2 (0,t,0,0),
// stride3 (t,0,0,0), random (w cells of w^4, domain 2) or malicious (RAW/RAS stride1, 1P stride2,
// R1P/3P the paper's groups of the 6 permutations of (x,y,z)).  Congestion: the
// warp ballot evaluator of rap_warp.cuh with merged duplicate cells.
#include <cuda_runtime.h>
#include <stdint.h>

#include "rap_rng.cuh"
#include "rap_warp.cuh"
#include "rap_internal.h"

namespace rapk {

constexpr int kSweep4Warps = 8;
constexpr int kMaxBins4 = 6 * 5 * (RAP_MAX_W + 1);
constexpr uint32_t kDomainQ = 3, kDomainR = 4;

// x mod w / x div w: masks and shifts when w is a compile-time power of two (W = 16, 32)
template <int W>
__device__ __forceinline__ uint32_t md(uint32_t x, uint32_t w) { return (W && !(W & (W - 1))) ? (x & (W - 1)) : x % w; }
template <int W>
__device__ __forceinline__ uint32_t dv(uint32_t x, uint32_t w) {
    return (W && !(W & (W - 1))) ? (x >> __builtin_ctz(W ? W : 1)) : x / w;
}

template <int W>
__global__ void __launch_bounds__(kSweep4Warps * 32)
sweep4_kernel(uint32_t w_rt, uint32_t pmask, uint32_t smask, uint64_t seed, uint64_t first, uint64_t n_trials,
              uint64_t *__restrict__ hist) {
    const uint32_t w = W ? (uint32_t)W : w_rt;
    __shared__ uint32_t sh_hist[kMaxBins4];
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    const uint32_t nbins = __popc(pmask) * __popc(smask) * (w + 1);
    for (uint32_t b = threadIdx.x; b < nbins; b += blockDim.x) sh_hist[b] = 0;
    __syncthreads();
    const LaneSel ls(lane);
    const uint32_t active = (w >= 32) ? kFull : ((1u << w) - 1u);
    const bool need_p = smask & ((1u << RAP_SCHEME4_1P) | (1u << RAP_SCHEME4_R1P) | (1u << RAP_SCHEME4_3P));
    const bool need_qr = (smask >> RAP_SCHEME4_3P) & 1u;
    const uint64_t stride = (uint64_t)gridDim.x * kSweep4Warps;
    for (uint64_t it = (uint64_t)blockIdx.x * kSweep4Warps + warp; it < n_trials; it += stride) {
        const uint64_t n = first + it;
        const uint32_t P = need_p ? warp_perm<W == 32 ? 32 : 0>(seed, n, lane, w) : lane;
        const uint32_t Q = need_qr ? warp_fisher_yates<W == 32 ? 32 : 0>(lane_word(seed, n, kDomainQ, lane), lane, w) : lane;
        const uint32_t R = need_qr ? warp_fisher_yates<W == 32 ? 32 : 0>(lane_word(seed, n, kDomainR, lane), lane, w) : lane;
        uint32_t cell_rnd = 0;
        if ((pmask >> RAP_PAT4_RANDOM) & 1u) {
            const uint64_t w4 = (uint64_t)w * w * w * w;
            cell_rnd = (uint32_t)(((uint64_t)lane_word(seed, n, kDomainRandom, lane) * w4) >> 32);
        }
        uint32_t mine = 0, e = 0;
        uint32_t c_s1[5] = {0, 0, 0, 0, 0}, c_s2[5] = {0, 0, 0, 0, 0};   // stride1 / stride2 results
        for (int p = 0; p < 6; ++p) {
            if (!((pmask >> p) & 1u)) continue;
            for (int s = 0; s < 5; ++s) {
                if (!((smask >> s) & 1u)) continue;
                int pp = p;
                if (p == RAP_PAT4_MALICIOUS)
                    pp = (s == RAP_SCHEME4_RAW || s == RAP_SCHEME4_RAS) ? RAP_PAT4_STRIDE1
                       : (s == RAP_SCHEME4_1P) ? RAP_PAT4_STRIDE2 : -1;
                // malicious = an access already evaluated this trial (reading xiii): reuse it
                if (p == RAP_PAT4_MALICIOUS && ((pp == RAP_PAT4_STRIDE1 && ((pmask >> RAP_PAT4_STRIDE1) & 1u)) ||
                                                (pp == RAP_PAT4_STRIDE2 && ((pmask >> RAP_PAT4_STRIDE2) & 1u)))) {
                    const uint32_t c = pp == RAP_PAT4_STRIDE1 ? c_s1[s] : c_s2[s];
                    mine = (lane == e) ? c : mine;
                    ++e;
                    continue;
                }
                uint32_t i = 0, j = 0, k = 0, l = 0;
                switch (pp) {
                case RAP_PAT4_CONTIGUOUS: l = lane; break;
                case RAP_PAT4_STRIDE1: k = lane; break;
                case RAP_PAT4_STRIDE2: j = lane; break;
                case RAP_PAT4_STRIDE3: i = lane; break;
                case RAP_PAT4_RANDOM: {
                    uint32_t c = cell_rnd;
                    l = md<W>(c, w); c = dv<W>(c, w);
                    k = md<W>(c, w); c = dv<W>(c, w);
                    j = md<W>(c, w); i = dv<W>(c, w);
                    break;
                }
                default: {                                          // 6-permutation groups
                    uint32_t g = lane / 6, m = lane % 6;
                    if (g >= w / 6 || 3 * g + 2 >= w) { g = 0; m = 0; }
                    const uint32_t v0 = 3 * g, v1 = 3 * g + 1, v2 = 3 * g + 2;
                    // (i,j,k) = the m-th permutation of (v0, v1, v2) in lexicographic order
                    const uint32_t a0 = m < 2 ? v0 : m < 4 ? v1 : v2;
                    const uint32_t a1 = (m == 0 || m == 5) ? v1 : (m == 1 || m == 3) ? v2 : v0;
                    i = a0; j = a1; k = 3 * g + 3 * g + 3 * g + 3 - a0 - a1;
                    l = 0;
                    break;
                }
                }
                // only the shuffles this scheme needs (s is warp-uniform)
                uint32_t f = 0;
                if (s == RAP_SCHEME4_RAS) {
                    f = mulshift(word_at(seed, n, kDomainRAS, (i * w + j) * w + k), w);
                } else if (s == RAP_SCHEME4_1P) {
                    f = __shfl_sync(kFull, P, k & 31u);
                } else if (s == RAP_SCHEME4_R1P) {
                    f = md<W>(__shfl_sync(kFull, P, i & 31u) + __shfl_sync(kFull, P, j & 31u) +
                              __shfl_sync(kFull, P, k & 31u), w);
                } else if (s == RAP_SCHEME4_3P) {
                    f = md<W>(__shfl_sync(kFull, P, i & 31u) + __shfl_sync(kFull, Q, j & 31u) +
                              __shfl_sync(kFull, R, k & 31u), w);
                }
                const uint32_t bank = md<W>(l + f, w);
                // merged requests: only the random cells and the clamped 6-permutation groups can
                // repeat a cell; every other pattern's w cells are distinct
                uint32_t counted = active;
                if (pp == RAP_PAT4_RANDOM || pp == -1) {
                    const uint32_t key = ((i * w + j) * w + k) * w + l;  // logical cell, < 2^20
                    const uint32_t same = __match_any_sync(kFull, lane < w ? key : (0x80000000u | lane));
                    counted = ballot_zero(same, (1u << lane) - 1u) & active;
                }
                const uint32_t c = max_bank_load(bank, counted, ls);
                if (p == RAP_PAT4_STRIDE1) c_s1[s] = c;
                if (p == RAP_PAT4_STRIDE2) c_s2[s] = c;
                mine = (lane == e) ? c : mine;
                ++e;
            }
        }
        if (lane < e) atomicAdd(&sh_hist[lane * (w + 1) + mine], 1u);
    }
    __syncthreads();
    for (uint32_t b = threadIdx.x; b < nbins; b += blockDim.x)
        if (sh_hist[b]) atomicAdd((unsigned long long *)(hist + b), (unsigned long long)sh_hist[b]);
}

cudaError_t launch_sweep4(uint32_t w, uint32_t pmask, uint32_t smask, uint64_t seed, uint64_t first,
                          uint64_t n_trials, uint64_t *hist, cudaStream_t st) {
    if (n_trials == 0) return cudaSuccess;
    int dev = 0, sms = 148, occ = 1;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    auto k = w == 32 ? sweep4_kernel<32> : w == 16 ? sweep4_kernel<16> : sweep4_kernel<0>;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k, kSweep4Warps * 32, 0);
    if (occ < 1) occ = 1;
    const uint64_t want = (n_trials + kSweep4Warps - 1) / kSweep4Warps;
    const uint64_t cap = (uint64_t)sms * occ;
    const int grid = (int)(want < cap ? want : cap);
    const uint64_t chunk = (uint64_t)grid * (1ull << 31) / 32;    // u32 CTA counters
    for (uint64_t done = 0; done < n_trials; done += chunk) {
        const uint64_t cnt = (n_trials - done < chunk) ? n_trials - done : chunk;
        k<<<grid, kSweep4Warps * 32, 0, st>>>(w, pmask, smask, seed, first + done, cnt, hist);
    }
    return cudaGetLastError();
}

}  // namespace rapk
