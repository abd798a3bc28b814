// exchange.cu -- step T4 of the RAP hot path (BASELINE cfg5): the block unpack that follows the
// NCCL all-to-all of the row-block-sharded transpose.  After rank g has transposed its M x N
// row block (rap_transpose) and exchanged the M x M blocks, block s of the receive buffer is
// (A[sM:(s+1)M, gM:(g+1)M])^T and belongs at columns sM..(s+1)M of the rank's output rows:
//     out[x * ld_out + s*M + a] = recv[(s*M + x) * M + a],   0 <= s < G, 0 <= x, a < M.
// A bandwidth-bound copy: 128-bit loads and stores when M and the pointers allow, one CTA per
// receive row at a time, persistent grid.
#include <cuda_runtime.h>
#include <stdint.h>

#include "rap_internal.h"

namespace rapk {

// V = vector type; each block has M rows of Mv vectors; ld_v = output row pitch in vectors.
// A CTA copies one receive row (s*M + x) at a time -- one division per row, not per element --
// with U independent vector loads per thread in flight before the stores.
constexpr int kUnpackThreads = 256, kUnpackU = 4;

template <typename V>
__global__ void __launch_bounds__(kUnpackThreads) unpack_blocks_kernel(const V *__restrict__ recv, V *__restrict__ out,
                                                                       int64_t G, int64_t M, int64_t Mv, int64_t ld_v) {
    const int64_t rows = G * M;
    for (int64_t row = blockIdx.x; row < rows; row += gridDim.x) {
        const int64_t s = row / M, x = row - s * M;
        const V *src = recv + row * Mv;
        V *dst = out + x * ld_v + s * Mv;
        for (int64_t a = threadIdx.x; a < Mv; a += (int64_t)kUnpackThreads * kUnpackU) {
            V v[kUnpackU];
#pragma unroll
            for (int u = 0; u < kUnpackU; ++u) {
                const int64_t idx = a + (int64_t)u * kUnpackThreads;
                if (idx < Mv) v[u] = __ldg(src + idx);
            }
#pragma unroll
            for (int u = 0; u < kUnpackU; ++u) {
                const int64_t idx = a + (int64_t)u * kUnpackThreads;
                if (idx < Mv) dst[idx] = v[u];
            }
        }
    }
}

cudaError_t launch_unpack_blocks(const void *recv, void *out, int64_t G, int64_t M, int64_t ld_out,
                                 uint32_t elem_bytes, cudaStream_t st) {
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    int64_t want = G * M;                                 // one CTA per receive row at most
    const int grid = (int)(want < (int64_t)sms * 8 ? want : (int64_t)sms * 8);
    const int64_t vb = 16;
    const bool v16 = ((uintptr_t)recv % 16 == 0) && ((uintptr_t)out % 16 == 0) &&
                     ((M * elem_bytes) % vb == 0) && ((ld_out * elem_bytes) % vb == 0);
    if (v16) {
        const int64_t k = vb / elem_bytes;
        unpack_blocks_kernel<uint4><<<grid, kUnpackThreads, 0, st>>>((const uint4 *)recv, (uint4 *)out, G, M, M / k,
                                                          ld_out / k);
    } else if (elem_bytes == 8) {
        unpack_blocks_kernel<uint64_t><<<grid, kUnpackThreads, 0, st>>>((const uint64_t *)recv, (uint64_t *)out, G, M, M,
                                                             ld_out);
    } else {
        unpack_blocks_kernel<uint32_t><<<grid, kUnpackThreads, 0, st>>>((const uint32_t *)recv, (uint32_t *)out, G, M, M,
                                                             ld_out);
    }
    return cudaGetLastError();
}

}  // namespace rapk
