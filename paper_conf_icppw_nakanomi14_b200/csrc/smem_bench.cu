// smem_bench.cu -- NEXT-1: the paper's own experiment (Table III, §VI) on B200.
//
// One CTA of 1024 threads = 32 warps transposes a 32 x 32 matrix between two shared-memory
// arrays a and b, `reps` times (a -> b, b -> a, ...), with the three algorithms of §III
// (P:L787-828): CRSW (contiguous read, stride write), SRCW (stride read, contiguous write) and
// DRDW (diagonal read, diagonal write), each under the RAW, RAS or RAP layout.  Both arrays carry
// the layout (reading v: the printed RAP listing P:L1521-1526 would write b column-wise with a
// 32-way conflict, contradicting Table III's write congestion 1).  Block k uses
// P = perm(seed, k, 32) / r = shifts(seed, k, 32), so averaging over many blocks measures the
// EXPECTED congestion; ncu's shared wavefronts per request is the hardware's congestion.
// Thread (i, j) = (tid / 32, tid % 32) performs, for the source array s and destination d:
//   CRSW  d[j][i]            <- s[i][j]
//   SRCW  d[i][j]            <- s[j][i]
//   DRDW  d[j][(i+j) mod 32] <- s[(i+j) mod 32][j] (reconstructed reading)
// Element (row, col) of an array lives at row*32 + ((col + sh[row]) mod 32); sh = 0 (RAW),
// r (RAS) or P (RAP).  Values are logical indices, so the result can be checked exactly.
#include <cuda_runtime.h>
#include <stdint.h>

#include "rap_rng.cuh"
#include "rap_internal.h"

namespace rapk {

template <int SCH>
__device__ __forceinline__ uint32_t sm_index(uint32_t row, uint32_t col, const uint32_t *sh) {
    if (SCH == RAP_SCHEME_RAW) return row * 32u + col;
    return row * 32u + ((col + sh[row]) & 31u);
}

template <int ALG, int SCH, typename T>
__global__ void __launch_bounds__(1024, 1)
smem_transpose_kernel(uint64_t seed, uint32_t reps, uint32_t *__restrict__ out, uint64_t *__restrict__ cycles) {
    __shared__ T a[1024], b[1024];
    __shared__ uint32_t sh[32];
    const uint32_t tid = threadIdx.x, i = tid >> 5, j = tid & 31u;
    if (i == 0) {
        uint32_t s = 0;
        if (SCH == RAP_SCHEME_RAP) s = warp_perm<32>(seed, blockIdx.x, j, 32);
        if (SCH == RAP_SCHEME_RAS) s = warp_ras_shift(seed, blockIdx.x, j, 32);
        sh[j] = s;
    }
    __syncthreads();
    a[sm_index<SCH>(i, j, sh)] = (T)(i * 32u + j);              // logical a[i][j] = i*32 + j
    __syncthreads();
    // the two addresses are loop-invariant: only the data accesses run inside the timed loop
    const uint32_t d = (i + j) & 31u;
    const uint32_t rd = ALG == 0 ? sm_index<SCH>(i, j, sh) : ALG == 1 ? sm_index<SCH>(j, i, sh) : sm_index<SCH>(d, j, sh);
    const uint32_t wr = ALG == 0 ? sm_index<SCH>(j, i, sh) : ALG == 1 ? sm_index<SCH>(i, j, sh) : sm_index<SCH>(j, d, sh);
    T *src = a, *dst = b;
    long long t0 = 0;
    if (tid == 0) t0 = clock64();
    for (uint32_t k = 0; k < reps; ++k) {
        dst[wr] = src[rd];
        __syncthreads();
        T *tmp = src; src = dst; dst = tmp;
    }
    if (tid == 0) cycles[blockIdx.x] = (uint64_t)(clock64() - t0);
    out[(size_t)blockIdx.x * 1024 + tid] = (uint32_t)src[sm_index<SCH>(i, j, sh)];   // logical (i, j)
}

// ------------------------------------------------------------------ NEXT-4: data-dependent access
// The paper's motivation: when the addresses a warp touches are not
// known beforehand, deterministic layouts have malicious inputs and RAP does not.  Here one CTA
// applies a permutation of the 32 x 32 tile `reps` times inside shared memory:
//     d[o / 32][o % 32] <- s[src[o] / 32][src[o] % 32]   for o = 0..1023 (thread o),
// a contiguous write and a data-dependent gather read, under layout RAW / PAD ([32][33]) /
// XOR ([i][j ^ i]) / RAS / RAP ([i][(j + sh[i]) mod 32]).  Warp s's read congestion is the DMM
// congestion of the 32 cells {src[32 s + t]} under the layout.
template <int L>
__device__ __forceinline__ uint32_t lay_index(uint32_t row, uint32_t col, const uint32_t *sh) {
    if (L == RAP_LAYOUT_PAD) return row * 33u + col;
    if (L == RAP_LAYOUT_XOR) return row * 32u + (col ^ row);
    if (L == RAP_LAYOUT_RAS || L == RAP_LAYOUT_RAP) return row * 32u + ((col + sh[row]) & 31u);
    return row * 32u + col;
}

template <int L>
__global__ void __launch_bounds__(1024, 1)
smem_gather_kernel(const uint16_t *__restrict__ src_index, uint64_t seed, uint32_t reps,
                   uint32_t *__restrict__ out, uint64_t *__restrict__ cycles) {
    __shared__ uint32_t a[32 * 33], b[32 * 33];
    __shared__ uint32_t sh[32];
    const uint32_t tid = threadIdx.x, i = tid >> 5, j = tid & 31u;
    if (i == 0) {
        uint32_t s = 0;
        if (L == RAP_LAYOUT_RAP) s = warp_perm<32>(seed, blockIdx.x, j, 32);
        if (L == RAP_LAYOUT_RAS) s = warp_ras_shift(seed, blockIdx.x, j, 32);
        sh[j] = s;
    }
    __syncthreads();
    a[lay_index<L>(i, j, sh)] = i * 32u + j;
    // indices >= 1024 are reduced mod 1024 on the device (the host cannot see device data; an
    // out-of-range index must not address past the tile, include/rap.h)
    const uint32_t g = src_index[tid] & 1023u;
    const uint32_t rd = lay_index<L>(g >> 5, g & 31u, sh);
    const uint32_t wr = lay_index<L>(i, j, sh);
    __syncthreads();
    uint32_t *srcb = a, *dstb = b;
    long long t0 = 0;
    if (tid == 0) t0 = clock64();
    for (uint32_t k = 0; k < reps; ++k) {
        dstb[wr] = srcb[rd];
        __syncthreads();
        uint32_t *tmp = srcb; srcb = dstb; dstb = tmp;
    }
    if (tid == 0) cycles[blockIdx.x] = (uint64_t)(clock64() - t0);
    out[(size_t)blockIdx.x * 1024 + tid] = srcb[wr];
}

cudaError_t launch_smem_gather(const uint16_t *src_index, int layout, uint64_t seed, uint32_t n_blocks,
                               uint32_t reps, uint32_t *out, uint64_t *cycles, cudaStream_t st) {
    switch (layout) {
    case RAP_LAYOUT_RAW: smem_gather_kernel<RAP_LAYOUT_RAW><<<n_blocks, 1024, 0, st>>>(src_index, seed, reps, out, cycles); break;
    case RAP_LAYOUT_PAD: smem_gather_kernel<RAP_LAYOUT_PAD><<<n_blocks, 1024, 0, st>>>(src_index, seed, reps, out, cycles); break;
    case RAP_LAYOUT_XOR: smem_gather_kernel<RAP_LAYOUT_XOR><<<n_blocks, 1024, 0, st>>>(src_index, seed, reps, out, cycles); break;
    case RAP_LAYOUT_RAS: smem_gather_kernel<RAP_LAYOUT_RAS><<<n_blocks, 1024, 0, st>>>(src_index, seed, reps, out, cycles); break;
    case RAP_LAYOUT_RAP: smem_gather_kernel<RAP_LAYOUT_RAP><<<n_blocks, 1024, 0, st>>>(src_index, seed, reps, out, cycles); break;
    default: return cudaErrorInvalidValue;
    }
    return cudaGetLastError();
}

cudaError_t launch_smem_bench(uint32_t alg, int scheme, uint32_t elem_bytes, uint64_t seed, uint32_t n_blocks,
                              uint32_t reps, uint32_t *out, uint64_t *cycles, cudaStream_t st) {
#define RAPK_SB(A, S)                                                                              \
    if (alg == A && scheme == S) {                                                                 \
        if (elem_bytes == 4) smem_transpose_kernel<A, S, uint32_t><<<n_blocks, 1024, 0, st>>>(seed, reps, out, cycles); \
        else smem_transpose_kernel<A, S, uint64_t><<<n_blocks, 1024, 0, st>>>(seed, reps, out, cycles);                 \
        return cudaGetLastError();                                                                 \
    }
    RAPK_SB(0, RAP_SCHEME_RAW) RAPK_SB(0, RAP_SCHEME_RAS) RAPK_SB(0, RAP_SCHEME_RAP)
    RAPK_SB(1, RAP_SCHEME_RAW) RAPK_SB(1, RAP_SCHEME_RAS) RAPK_SB(1, RAP_SCHEME_RAP)
    RAPK_SB(2, RAP_SCHEME_RAW) RAPK_SB(2, RAP_SCHEME_RAS) RAPK_SB(2, RAP_SCHEME_RAP)
#undef RAPK_SB
    return cudaErrorInvalidValue;
}

}  // namespace rapk
