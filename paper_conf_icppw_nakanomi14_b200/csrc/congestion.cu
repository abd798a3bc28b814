// congestion.cu -- steps C1-C4 of the RAP hot path: the DMM congestion evaluator and its
// Monte-Carlo sweep (Table II, §V), plus the batched evaluator,
// the trace evaluator and the device permutation generator (T0).
//
// One CUDA warp simulates one DMM warp of w <= 32 threads (§II): lane t issues the
// request of DMM thread t.  Congestion: requests to the same address are merged
// (__match_any_sync on the address, one leader per address), then the number of distinct
// requests per bank is popc(__match_any_sync(bank)) and the congestion is the warp maximum
// (__reduce_max_sync).  Permutations come from a warp Fisher-Yates shuffle (rap_rng.cuh);
// P[i] and r[i] stay in lane i's register and are read with __shfl_sync(., row).
// Histograms: warp-private u32 counters in shared memory (no atomics: evaluation e is
// counted by lane e), reduced per CTA and added once to the caller's u64 bins.
#include <cuda_runtime.h>
#include <stdint.h>

#include "rap_rng.cuh"
#include "rap_internal.h"

namespace rapk {

constexpr int kSweepWarps = 8;
constexpr int kMaxEval = 25;                 // 5 patterns x 5 schemes
constexpr int kMaxBins = kMaxEval * (RAP_MAX_W + 1);

// Congestion of the warp access in which active lane t (< w) requests logical cell
// (row, col) of a w x w matrix stored by `scheme`.  P / r: lane i holds P[i] / r[i].
template <int W>
__device__ __forceinline__ uint32_t warp_congestion(uint32_t row, uint32_t col, int scheme, uint32_t P,
                                                    uint32_t r, uint32_t lane, uint32_t w_rt,
                                                    bool dedupe) {
    const uint32_t w = W ? (uint32_t)W : w_rt;
    const bool active = lane < w;
    uint32_t addr, bank;
    switch (scheme) {
    case RAP_SCHEME_RAS:
    case RAP_SCHEME_RAP: {
        const uint32_t sh = __shfl_sync(kFull, scheme == RAP_SCHEME_RAP ? P : r, row & 31u);
        uint32_t pc = col + sh;
        pc = (pc >= w) ? pc - w : pc;                    // (col + shift[row]) mod w
        bank = pc;
        addr = row * w + pc;
        break;
    }
    case RAP_SCHEME_PAD: {
        uint32_t b = row + col;
        bank = (b >= w) ? b - w : b;                     // (row*(w+1) + col) mod w
        addr = row * (w + 1) + col;
        break;
    }
    case RAP_SCHEME_XOR:
        bank = col ^ row;
        addr = row * w + bank;
        break;
    default:                                             // RAW
        bank = col;
        addr = row * w + col;
        break;
    }
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

// ------------------------------------------------------------------ C1-C4 sweep
template <int W>
__global__ void __launch_bounds__(kSweepWarps * 32)
sweep_kernel(uint32_t w_rt, uint32_t pmask, uint32_t smask, uint64_t seed, uint64_t first,
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
        // C1: lane L computes Philox block (L & 7) of domain (L >> 3): 24 useful blocks
        const uint4 blk = philox_block(seed, n, lane >> 3, lane & 7u);
        *reinterpret_cast<uint4 *>(&sh_words[warp][4 * lane]) = blk;   // word(d,t) at [32d + t]
        __syncwarp();
        const uint32_t u_fy = sh_words[warp][lane];
        const uint32_t u_ras = sh_words[warp][32 + lane];
        const uint32_t u_rnd = sh_words[warp][64 + lane];
        __syncwarp();
        // C2: warp Fisher-Yates; RAS shifts; random cells
        const uint32_t P = warp_fisher_yates<W>(u_fy, lane, w);
        const uint32_t r = mulshift(u_ras, w);
        uint32_t rrow = 0, rcol = 0;
        if (any_random) {
            const uint32_t cell = mulshift(u_rnd, w * w);
            if (W == 32) { rrow = cell >> 5; rcol = cell & 31u; }
            else { rrow = cell / w; rcol = cell - rrow * w; }
        }
        // C3: every selected (pattern, scheme); lane e keeps evaluation e's congestion
        uint32_t mine = 0, e = 0;
#pragma unroll
        for (int p = 0; p < 5; ++p) {
            if (!((pmask >> p) & 1u)) continue;
#pragma unroll
            for (int s = 0; s < 5; ++s) {
                if (!((smask >> s) & 1u)) continue;
                uint32_t row, col;
                pattern_cell(p, s, lane, w, rrow, rcol, row, col);
                const uint32_t c = warp_congestion<W>(row, col, s, P, r, lane, w, p == RAP_PAT_RANDOM);
                mine = (lane == e) ? c : mine;
                ++e;
            }
        }
        // C4: count
        if (lane < e) sh_hist[warp][lane * (w + 1) + mine] += 1;
    }
    flush_hist(sh_hist, kSweepWarps, nbins, hist);
}

// ------------------------------------------------------------------ trace evaluator
constexpr int kTraceChunk = 32;

__global__ void __launch_bounds__(kSweepWarps * 32)
trace_kernel(uint32_t w, uint64_t n_warps, const uint32_t *__restrict__ cells, uint32_t smask,
             uint64_t seed, uint64_t first, uint64_t n_trials, uint64_t *__restrict__ hist) {
    __shared__ uint32_t sh_hist[kSweepWarps][kMaxBins];
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    const uint32_t nsch = __popc(smask);
    const uint32_t nbins = nsch * (w + 1);
    for (uint32_t b = lane; b < nbins; b += 32) sh_hist[warp][b] = 0;
    __syncwarp();
    const bool need_p = (smask >> RAP_SCHEME_RAP) & 1u, need_r = (smask >> RAP_SCHEME_RAS) & 1u;
    const uint64_t nchunks = (n_warps + kTraceChunk - 1) / kTraceChunk;
    const uint64_t nitems = n_trials * nchunks;
    const uint64_t stride = (uint64_t)gridDim.x * kSweepWarps;
    for (uint64_t it = (uint64_t)blockIdx.x * kSweepWarps + warp; it < nitems; it += stride) {
        const uint64_t trial = it / nchunks, chunk = it - trial * nchunks;
        const uint64_t n = first + trial;
        const uint32_t P = need_p ? warp_perm<0>(seed, n, lane, w) : lane;
        const uint32_t r = need_r ? warp_ras_shift(seed, n, lane, w) : 0u;
        const uint64_t k_end = min(n_warps, (chunk + 1) * kTraceChunk);
        for (uint64_t k = chunk * kTraceChunk; k < k_end; ++k) {
            const uint32_t raw_cell = (lane < w) ? cells[k * w + lane] : 0u;
            const bool bad = __any_sync(kFull, raw_cell >= w * w);   // counted in bin 0
            const uint32_t cell = bad ? 0u : raw_cell;
            const uint32_t row = cell / w, col = cell - (cell / w) * w;
            uint32_t mine = 0, e = 0;
#pragma unroll
            for (int s = 0; s < 5; ++s) {
                if (!((smask >> s) & 1u)) continue;
                const uint32_t c = warp_congestion<0>(row, col, s, P, r, lane, w, true);
                mine = (lane == e) ? (bad ? 0u : c) : mine;
                ++e;
            }
            if (lane < e) sh_hist[warp][lane * (w + 1) + mine] += 1;
        }
    }
    flush_hist(sh_hist, kSweepWarps, nbins, hist);
}

// ------------------------------------------------------------------ batched evaluator
__global__ void __launch_bounds__(256)
congestion_kernel(uint32_t w, uint64_t n_warps, const uint32_t *__restrict__ rows,
                  const uint32_t *__restrict__ cols, int scheme, const uint32_t *__restrict__ shift,
                  uint32_t *__restrict__ out) {
    const uint32_t lane = threadIdx.x & 31u;
    const uint64_t stride = (uint64_t)gridDim.x * (blockDim.x >> 5);
    for (uint64_t k = (uint64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); k < n_warps;
         k += stride) {
        const bool active = lane < w;
        const uint32_t row = active ? rows[k * w + lane] : 0u;
        const uint32_t col = active ? cols[k * w + lane] : 0u;
        const uint32_t sh = (active && shift) ? shift[k * w + lane] : 0u;
        const bool bad = active && (row >= w || col >= w || sh >= w);
        const uint32_t c = warp_congestion<0>(active ? row % w : 0u, active ? col % w : 0u, scheme,
                                              sh % w, sh % w, lane, w, true);
        const bool any_bad = __any_sync(kFull, bad);
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
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    return sms;
}

template <typename K>
static int resident_ctas(K kernel, int threads) {
    int occ = 1;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kernel, threads, 0);
    return (occ < 1 ? 1 : occ) * sm_count();
}

static int clamp_grid(uint64_t items, int per_cta, int cap) {
    const uint64_t want = (items + per_cta - 1) / per_cta;
    return (int)(want < (uint64_t)cap ? (want ? want : 1) : (uint64_t)cap);
}

cudaError_t launch_sweep(uint32_t w, uint32_t pmask, uint32_t smask, uint64_t seed, uint64_t first,
                         uint64_t n_trials, uint64_t *hist, cudaStream_t st) {
    if (n_trials == 0) return cudaSuccess;
    const int threads = kSweepWarps * 32;
    if (w == 32) {
        auto k = sweep_kernel<32>;
        const int grid = clamp_grid(n_trials, kSweepWarps, resident_ctas(k, threads));
        // per-warp u32 counters: keep trials per warp below 2^31 by chunking the range
        const uint64_t chunk = (uint64_t)grid * kSweepWarps * (1ull << 31);
        for (uint64_t done = 0; done < n_trials; done += chunk) {
            const uint64_t cnt = (n_trials - done < chunk) ? n_trials - done : chunk;
            k<<<grid, threads, 0, st>>>(w, pmask, smask, seed, first + done, cnt, hist);
        }
    } else {
        auto k = sweep_kernel<0>;
        const int grid = clamp_grid(n_trials, kSweepWarps, resident_ctas(k, threads));
        const uint64_t chunk = (uint64_t)grid * kSweepWarps * (1ull << 31);
        for (uint64_t done = 0; done < n_trials; done += chunk) {
            const uint64_t cnt = (n_trials - done < chunk) ? n_trials - done : chunk;
            k<<<grid, threads, 0, st>>>(w, pmask, smask, seed, first + done, cnt, hist);
        }
    }
    return cudaGetLastError();
}

cudaError_t launch_trace(uint32_t w, uint64_t n_warps, const uint32_t *cells, uint32_t smask,
                         uint64_t seed, uint64_t first, uint64_t n_trials, uint64_t *hist,
                         cudaStream_t st) {
    if (n_trials == 0 || n_warps == 0) return cudaSuccess;
    const int threads = kSweepWarps * 32;
    const uint64_t nchunks = (n_warps + kTraceChunk - 1) / kTraceChunk;
    const int grid = clamp_grid(n_trials * nchunks, kSweepWarps, resident_ctas(trace_kernel, threads));
    // counts per warp <= items_per_warp * kTraceChunk; chunk the trial range to stay < 2^31
    const uint64_t trials_chunk = ((uint64_t)grid * kSweepWarps * ((1ull << 31) / kTraceChunk)) / nchunks + 1;
    for (uint64_t done = 0; done < n_trials; done += trials_chunk) {
        const uint64_t cnt = (n_trials - done < trials_chunk) ? n_trials - done : trials_chunk;
        trace_kernel<<<grid, threads, 0, st>>>(w, n_warps, cells, smask, seed, first + done, cnt, hist);
    }
    return cudaGetLastError();
}

cudaError_t launch_congestion(uint32_t w, uint64_t n_warps, const uint32_t *rows, const uint32_t *cols,
                              int scheme, const uint32_t *shift, uint32_t *out, cudaStream_t st) {
    if (n_warps == 0) return cudaSuccess;
    const int grid = clamp_grid(n_warps, 8, resident_ctas(congestion_kernel, 256));
    congestion_kernel<<<grid, 256, 0, st>>>(w, n_warps, rows, cols, scheme, shift, out);
    return cudaGetLastError();
}

cudaError_t launch_perm_gen(uint64_t seed, uint64_t first, uint64_t count, uint32_t w, uint8_t *out,
                            cudaStream_t st) {
    if (count == 0) return cudaSuccess;
    const int grid = clamp_grid(count, 8, resident_ctas(perm_gen_kernel, 256));
    perm_gen_kernel<<<grid, 256, 0, st>>>(seed, first, count, w, out);
    return cudaGetLastError();
}

}  // namespace rapk
