// sweep_wide.cu -- NEXT-3: the congestion sweep for DMMs wider than a CUDA warp, 32 < w <= 256
// (Table II's w = 64, 128, 256 columns, §V; "the value of w may be increased in
// future GPUs").
//
// A DMM warp of w > 32 threads does not fit one CUDA warp, so here ONE CUDA THREAD SIMULATES ONE
// TRIAL: it draws its permutation (Durstenfeld on a private array), its RAS shifts and its random
// cells from the same counter contract as every other kernel (rap_rng.cuh / include/rap.h), then
// walks the w requests of each (pattern, scheme), counting distinct requests per bank in a private
// array.  Private arrays live in shared memory laid out [index][thread] (element k of thread t at
// k*T + t), so at any step the T threads of a CTA touch T consecutive 16-bit slots: no bank
// conflicts whatever index each thread uses.  Merged requests (random cells) are found once per
// trial: a request is a leader if no earlier request of the trial has the same cell.
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

size_t wide_smem_bytes(uint32_t w, uint32_t pmask, uint32_t smask) {
    const uint32_t nbins = __builtin_popcount(pmask) * __builtin_popcount(smask) * (w + 1);
    return 4 * (size_t)((nbins + 3) & ~3u) + 2 * (size_t)4 * w * kWideThreads +
           4 * (size_t)((w + 31) / 32) * kWideThreads;
}

cudaError_t launch_sweep_wide(uint32_t w, uint32_t pmask, uint32_t smask, uint64_t seed, uint64_t first,
                              uint64_t n_trials, uint64_t *hist, cudaStream_t st) {
    if (n_trials == 0) return cudaSuccess;
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

}  // namespace rapk
