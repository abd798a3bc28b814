// transpose_rap16.cu -- T2b option (ii): the 64-bit transpose on a tile of doubles laid out
// RAP-16 (RAP_LAYOUT_RAP16), the ablation of the two-plane design in transpose.cu.
//
// The paper assumed one double per bank word.  B200 has 32 banks of 4 bytes,
// so a double occupies a PAIR of banks and a warp-wide 64-bit shared access moves 256 bytes: at
// least 2 wavefronts, each serving 16 lanes with 16 distinct bank pairs at best.  RAP-16 is the
// paper's RAP with w = 16 "double banks" applied to each half of a row:
//     a[i][j] at [i][16 * (j div 16) + ((j + Q[i mod 16]) mod 16)],   Q = perm(seed, 0, 16)
// (reading xiv).  A row (contiguous) access by lanes j = 0..15 hits double banks
// (j + Q[i]) mod 16 -- distinct; a column (stride) access by lanes i = 0..15 (or 16..31) hits
// (c + Q[i mod 16]) mod 16 -- distinct because Q is a permutation (Theorem 2's argument at
// w = 16).  So every LDS.64 / STS.64 should take the ideal 2 wavefronts.
//
// Kernel shape (as transpose.cu): one warp per 32 x 32 tile, a CTA of SR warps stacked along
// the input rows drains in lockstep, persistent CTAs, one tile of loads in flight.
//   load  : LDG.64, lane j reads element j of each of the 32 tile rows (256 B per row)
//   smem  : STS.64 at double i*64 + 32*(j div 16) + (j mod 16) + Q[i mod 16]  (unwrapped
//           16-double windows, the bank decoder performs the "mod 16"; base + immediate)
//   drain : lane i reads column c at i*64 + Q[i mod 16] + c (+16 for c >= 16): LDS.64, then
//           output row c as one 256-byte STG.64
#include <cuda_runtime.h>
#include <stdint.h>

#include "rap_rng.cuh"
#include "rap_internal.h"

namespace rapk {

constexpr int kR16Pitch = 64;               // doubles per tile row (two unwrapped 32-double windows)
constexpr int kR16SR = 12;                  // warps (tiles) per CTA, stacked along input rows

template <int SR>
__global__ void __launch_bounds__(SR * 32, 1)
transpose_rap16_kernel(const uint2 *__restrict__ src, uint2 *__restrict__ dst, int64_t rows, int64_t cols,
                       int64_t ld_src, int64_t ld_dst, const TileShifts ts, uint32_t tiles_r, uint32_t tiles_c) {
    extern __shared__ __align__(16) uint2 smem_r16[];
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    uint2 *tile = smem_r16 + warp * (32 * kR16Pitch);

    // T0: lanes 0..15 hold Q[lane] (Durstenfeld at w = 16, domain 0, index 0; host, tile_shifts)
    const uint32_t qv = shift_byte(ts.sh, lane & 15u);
    // T1 offsets: lane j writes row i at i*64 + st_off[i mod 16]
    uint32_t st_off[16];
#pragma unroll
    for (int k = 0; k < 16; ++k) st_off[k] = 2u * (lane & 16u) + (lane & 15u) + __shfl_sync(kFull, qv, k);
    // T2 base: lane i reads row i, column c at drain_base + c (+ 16 for c >= 16)
    const uint32_t drain_base = lane * kR16Pitch + __shfl_sync(kFull, qv, lane & 15u);

    const uint32_t nst = ((tiles_r + SR - 1) / SR) * tiles_c;
    auto coords = [&](uint32_t st, uint32_t &ti, uint32_t &tj) -> bool {
        const uint32_t si = st / tiles_c;
        tj = st - si * tiles_c;
        ti = si * SR + warp;
        return ti < tiles_r;
    };
    auto load = [&](uint2 (&v)[32], uint32_t ti, uint32_t tj) {
        const int64_t r0 = (int64_t)ti * 32, c0 = (int64_t)tj * 32;
        const uint2 *p = src + r0 * ld_src + c0 + lane;
        if (r0 + 32 <= rows && c0 + 32 <= cols) {
#pragma unroll
            for (int r = 0; r < 32; ++r) v[r] = __ldg(p + (int64_t)r * ld_src);
        } else {
            const bool cok = c0 + lane < cols;
#pragma unroll
            for (int r = 0; r < 32; ++r)
                v[r] = (cok && r0 + r < rows) ? __ldg(p + (int64_t)r * ld_src) : make_uint2(0u, 0u);
        }
    };
    auto store_tile = [&](const uint2 (&v)[32]) {
#pragma unroll
        for (int r = 0; r < 32; ++r) tile[r * kR16Pitch + st_off[r & 15]] = v[r];
    };
    auto drain = [&](uint32_t ti, uint32_t tj) {
        const int64_t r0 = (int64_t)ti * 32, c0 = (int64_t)tj * 32;
        uint2 *o = dst + c0 * ld_dst + r0 + lane;
        if (r0 + 32 <= rows && c0 + 32 <= cols) {
#pragma unroll
            for (int c = 0; c < 32; ++c) {
                *o = tile[drain_base + c + (c >= 16 ? 16 : 0)];
                o += ld_dst;
            }
        } else {
            const bool rok = r0 + lane < rows;
            const int cmax = (int)min((int64_t)32, cols - c0);
#pragma unroll
            for (int c = 0; c < 32; ++c) {
                if (c < cmax && rok) *o = tile[drain_base + c + (c >= 16 ? 16 : 0)];
                o += ld_dst;
            }
        }
    };

    uint32_t st = blockIdx.x, ti = 0, tj = 0;
    bool act = st < nst && coords(st, ti, tj);
    uint2 v[32];
    if (!ts.early) pdl_wait(), pdl_trigger();                       // the previous grid's writes are visible
    if (act) load(v, ti, tj);
    if (ts.early) pdl_wait(), pdl_trigger();        // before the first global store
    while (st < nst) {
        const uint32_t cti = ti, ctj = tj;
        const bool cact = act;
        if (cact) store_tile(v);                     // T1
        __syncwarp();
        st += gridDim.x;
        act = st < nst && coords(st, ti, tj);
        if (act) load(v, ti, tj);                    // T3: next tile in flight
        if (SR > 1) __syncthreads();                 // drains of the super-tile together
        if (cact) drain(cti, ctj);                   // T2
        __syncwarp();
    }
}

cudaError_t launch_transpose_rap16(const void *src, void *dst, int64_t rows, int64_t cols, int64_t ld_src,
                                   int64_t ld_dst, uint64_t seed, cudaStream_t st) {
    constexpr int SR = kR16SR;
    auto k = transpose_rap16_kernel<SR>;
    const size_t smem = sizeof(uint2) * 32 * kR16Pitch * SR;
    static ShapeCache cache;
    const uint32_t tiles_r = (uint32_t)((rows + 31) / 32), tiles_c = (uint32_t)((cols + 31) / 32);
    const int64_t nst = (int64_t)((tiles_r + SR - 1) / SR) * tiles_c;
    int grid = 0;
    const cudaError_t e = cached_grid(k, cache, SR * 32, smem, nst, 0, &grid);
    if (e != cudaSuccess) return e;
    TileShifts ts = tile_shifts(RAP_LAYOUT_RAP16, seed);
    ts.early = pdl_early_loads(st, src, rows, cols, ld_src, dst, cols, rows, ld_dst, 8u) ? 1u : 0u;
    return launch_ex(k, grid, SR * 32, smem, st, 1, (const uint2 *)src, (uint2 *)dst, rows, cols, ld_src, ld_dst, ts,
                     tiles_r, tiles_c);
}

}  // namespace rapk
