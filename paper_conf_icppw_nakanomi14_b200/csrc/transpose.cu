// transpose.cu -- steps T0-T3 of the RAP hot path: the out-of-place HBM transpose staged
// through 32 x 32 shared-memory tiles laid out RAW / PAD / XOR / RAS / RAP.
//
// Paper: the RAP CRSW transpose of one 32 x 32 tile (§VI) moves a[i][j] to
// b[j][i] with a[i][j] stored at a[i][(j + P[i]) mod 32] (§IV), so that the
// row-wise (contiguous) write AND the column-wise (stride) read of the tile are both
// conflict-free for every P (Theorem 2).
//
// B200 design: one warp owns one 32 x 32 tile buffer (no CTA barrier,
// only __syncwarp), persistent warps stride over the tile grid, and the next tile's global
// loads are in flight while the current tile is drained.
//   load  : 128-bit LDG.  One warp instruction covers 4 tile rows x 128 B.  Under RAP the 4
//           rows are chosen as P^-1(4g+0..3), i.e. rows whose P values cover the 4 residues
//           mod 4, which makes each of the 4 following STS.32 hit 32 distinct banks:
//           bank(row, 4q+k) = (4q + k + 4g + c) mod 32 is injective in (c, q).
//   smem  : STS.32 of element (i, j) at column phys(i, j) of row i.
//   drain : lane i reads column c of the tile at phys(i, c): the DMM stride access, banks
//           (c + P[i]) mod 32 distinct because P is a permutation; then 128-byte coalesced
//           STG.32 of output row c.
// 64-bit elements: 32 banks of 4 bytes (the paper assumed one double per bank word,
// P:L278-283, L860), so a tile of doubles is split into two 32-bit RAP planes (low / high
// words) with identical addressing; every smem access stays a 32-lane 4-byte access.
#include <cuda_runtime.h>
#include <stdint.h>

#include "rap_rng.cuh"
#include "rap_internal.h"

namespace rapk {

template <int L>
struct Tile {
    static constexpr int S = (L == RAP_LAYOUT_PAD) ? 33 : 32;   // row pitch in 4-byte words
};

// physical column of logical element (row, col) of the tile; sh = shift of that row
template <int L>
__device__ __forceinline__ uint32_t phys_col(uint32_t row, uint32_t col, uint32_t sh) {
    if (L == RAP_LAYOUT_XOR) return col ^ row;
    if (L == RAP_LAYOUT_RAS || L == RAP_LAYOUT_RAP) return (col + sh) & 31u;
    return col;
}

__device__ __forceinline__ uint4 ldg_stream128(const void *p) {
    uint4 r;
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
    return r;
}

// Per-warp prologue shared by the 32- and 64-bit kernels: sh_lane = shift of tile row `lane`
// (P[lane] for RAP, r[lane] for RAS), and for load group g of G groups of R = 32/G rows the
// row this lane loads and that row's shift.
template <int L, int G>
__device__ __forceinline__ void tile_rows(uint32_t *scratch, uint64_t seed, uint32_t lane,
                                          uint32_t &sh_lane, uint32_t (&row_g)[G], uint32_t (&sh_g)[G]) {
    constexpr int R = 32 / G;                  // rows covered by one load instruction
    const uint32_t c = lane / (32 / R);        // which of the R rows this lane loads
    sh_lane = 0;
    if (L == RAP_LAYOUT_RAP) sh_lane = warp_perm<32>(seed, 0, lane, 32);
    if (L == RAP_LAYOUT_RAS) sh_lane = warp_ras_shift(seed, 0, lane, 32);
    if (L == RAP_LAYOUT_RAP) {
        scratch[sh_lane] = lane;               // P^-1 through shared memory
        __syncwarp();
        const uint32_t pinv = scratch[lane];
        __syncwarp();
#pragma unroll
        for (int g = 0; g < G; ++g) {
            row_g[g] = __shfl_sync(kFull, pinv, R * g + c);   // P[row_g] = R*g + c
            sh_g[g] = R * g + c;
        }
    } else {
#pragma unroll
        for (int g = 0; g < G; ++g) {
            row_g[g] = R * g + c;
            sh_g[g] = __shfl_sync(kFull, sh_lane, R * g + c);
        }
    }
}

// Tile t -> (ti, tj).  Tiles are walked in groups of `group` tile-rows, column by column
// inside a group, so the ~#warps tiles in flight at any moment form a roughly square block:
// both the input rows they read and the output rows they write are long contiguous runs
// (DRAM page locality on both sides).  group == 0: plain row-major tile order.
__device__ __forceinline__ void tile_coords(uint32_t t, uint32_t tiles_r, uint32_t tiles_c, uint32_t group,
                                            uint32_t &ti, uint32_t &tj) {
    if (group == 0) {
        ti = t / tiles_c;
        tj = t - ti * tiles_c;
        return;
    }
    const uint32_t per = group * tiles_c;
    const uint32_t g = t / per, rem = t - g * per;
    const uint32_t base = g * group;
    const uint32_t nrows = min(group, tiles_r - base);
    tj = rem / nrows;
    ti = base + (rem - tj * nrows);
}

// ------------------------------------------------------------------ 32-bit elements
constexpr int kWarps32 = 8;

template <int L, bool VEC, int MINB>
__global__ void __launch_bounds__(kWarps32 * 32, MINB)
transpose_b32_kernel(const uint32_t *__restrict__ src, uint32_t *__restrict__ dst, int64_t rows,
                     int64_t cols, int64_t ld_src, int64_t ld_dst, uint64_t seed, uint32_t tiles_r,
                     uint32_t tiles_c, uint32_t ntiles, uint32_t group) {
    constexpr int S = Tile<L>::S;
    __shared__ __align__(16) uint32_t smem[kWarps32][32 * S];
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    uint32_t *tile = smem[warp];

    uint32_t sh_lane, row_g[8], sh_g[8];
    tile_rows<L, 8>(tile, seed, lane, sh_lane, row_g, sh_g);
    const uint32_t q = lane & 7u;              // 16-byte chunk of the row

    const uint32_t stride = gridDim.x * kWarps32;
    uint32_t t = blockIdx.x * kWarps32 + warp;
    uint4 v[8];

    auto load = [&](uint32_t tt) {
        uint32_t ti, tj;
        tile_coords(tt, tiles_r, tiles_c, group, ti, tj);
        const int64_t r0 = (int64_t)ti * 32, c0 = (int64_t)tj * 32;
        const bool full = (r0 + 32 <= rows) && (c0 + 32 <= cols);
        if (VEC && full) {
#pragma unroll
            for (int g = 0; g < 8; ++g)
                v[g] = ldg_stream128(src + (r0 + row_g[g]) * ld_src + c0 + 4 * q);
        } else {
#pragma unroll
            for (int g = 0; g < 8; ++g) {
                const int64_t r = r0 + row_g[g];
                const uint32_t *p = src + r * ld_src + c0 + 4 * q;
                const bool rok = r < rows;
                const int64_t cc = c0 + 4 * q;
                v[g].x = (rok && cc + 0 < cols) ? __ldg(p + 0) : 0u;
                v[g].y = (rok && cc + 1 < cols) ? __ldg(p + 1) : 0u;
                v[g].z = (rok && cc + 2 < cols) ? __ldg(p + 2) : 0u;
                v[g].w = (rok && cc + 3 < cols) ? __ldg(p + 3) : 0u;
            }
        }
    };

    if (t < ntiles) load(t);
    while (t < ntiles) {
        // T1: contiguous (row-wise) write of the tile into shared memory
#pragma unroll
        for (int g = 0; g < 8; ++g) {
            uint32_t *rowp = tile + row_g[g] * S;
            rowp[phys_col<L>(row_g[g], 4 * q + 0, sh_g[g])] = v[g].x;
            rowp[phys_col<L>(row_g[g], 4 * q + 1, sh_g[g])] = v[g].y;
            rowp[phys_col<L>(row_g[g], 4 * q + 2, sh_g[g])] = v[g].z;
            rowp[phys_col<L>(row_g[g], 4 * q + 3, sh_g[g])] = v[g].w;
        }
        __syncwarp();
        const uint32_t cur = t;
        t += stride;
        if (t < ntiles) load(t);               // T3: next tile in flight while draining

        // T2: stride (column-wise) read of the tile, coalesced row writes of the output
        uint32_t ti, tj;
        tile_coords(cur, tiles_r, tiles_c, group, ti, tj);
        const int64_t r0 = (int64_t)ti * 32, c0 = (int64_t)tj * 32;
        const uint32_t *myrow = tile + lane * S;
        uint32_t *out = dst + c0 * ld_dst + r0 + lane;
        if ((r0 + 32 <= rows) && (c0 + 32 <= cols)) {
#pragma unroll
            for (int c = 0; c < 32; ++c) out[c * ld_dst] = myrow[phys_col<L>(lane, c, sh_lane)];
        } else {
            const bool rok = r0 + lane < rows;
            const int64_t cmax = cols - c0;
#pragma unroll 4
            for (int c = 0; c < 32; ++c)
                if (rok && c < cmax) out[c * ld_dst] = myrow[phys_col<L>(lane, c, sh_lane)];
        }
        __syncwarp();
    }
}

// ------------------------------------------------------------------ 64-bit elements
constexpr int kWarps64 = 4;

template <int L, bool VEC, int MINB>
__global__ void __launch_bounds__(kWarps64 * 32, MINB)
transpose_b64_kernel(const uint64_t *__restrict__ src, uint64_t *__restrict__ dst, int64_t rows,
                     int64_t cols, int64_t ld_src, int64_t ld_dst, uint64_t seed, uint32_t tiles_r,
                     uint32_t tiles_c, uint32_t ntiles, uint32_t group) {
    constexpr int S = Tile<L>::S;
    __shared__ __align__(16) uint32_t smem[kWarps64][2][32 * S];   // [warp][lo/hi plane]
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    uint32_t *lo_plane = smem[warp][0];
    uint32_t *hi_plane = smem[warp][1];

    uint32_t sh_lane, row_g[16], sh_g[16];
    tile_rows<L, 16>(lo_plane, seed, lane, sh_lane, row_g, sh_g);
    const uint32_t q = lane & 15u;             // 16-byte chunk = elements 2q, 2q+1

    const uint32_t stride = gridDim.x * kWarps64;
    uint32_t t = blockIdx.x * kWarps64 + warp;
    uint4 v[16];

    auto load = [&](uint32_t tt) {
        uint32_t ti, tj;
        tile_coords(tt, tiles_r, tiles_c, group, ti, tj);
        const int64_t r0 = (int64_t)ti * 32, c0 = (int64_t)tj * 32;
        const bool full = (r0 + 32 <= rows) && (c0 + 32 <= cols);
        if (VEC && full) {
#pragma unroll
            for (int g = 0; g < 16; ++g)
                v[g] = ldg_stream128(src + (r0 + row_g[g]) * ld_src + c0 + 2 * q);
        } else {
#pragma unroll
            for (int g = 0; g < 16; ++g) {
                const int64_t r = r0 + row_g[g];
                const uint64_t *p = src + r * ld_src + c0 + 2 * q;
                const bool rok = r < rows;
                const int64_t cc = c0 + 2 * q;
                const uint64_t e0 = (rok && cc + 0 < cols) ? __ldg((const unsigned long long *)p + 0) : 0ull;
                const uint64_t e1 = (rok && cc + 1 < cols) ? __ldg((const unsigned long long *)p + 1) : 0ull;
                v[g] = make_uint4((uint32_t)e0, (uint32_t)(e0 >> 32), (uint32_t)e1, (uint32_t)(e1 >> 32));
            }
        }
    };

    if (t < ntiles) load(t);
    while (t < ntiles) {
#pragma unroll
        for (int g = 0; g < 16; ++g) {
            const uint32_t p0 = row_g[g] * S + phys_col<L>(row_g[g], 2 * q + 0, sh_g[g]);
            const uint32_t p1 = row_g[g] * S + phys_col<L>(row_g[g], 2 * q + 1, sh_g[g]);
            lo_plane[p0] = v[g].x;
            hi_plane[p0] = v[g].y;
            lo_plane[p1] = v[g].z;
            hi_plane[p1] = v[g].w;
        }
        __syncwarp();
        const uint32_t cur = t;
        t += stride;
        if (t < ntiles) load(t);

        uint32_t ti, tj;
        tile_coords(cur, tiles_r, tiles_c, group, ti, tj);
        const int64_t r0 = (int64_t)ti * 32, c0 = (int64_t)tj * 32;
        const uint32_t *mylo = lo_plane + lane * S;
        const uint32_t *myhi = hi_plane + lane * S;
        uint64_t *out = dst + c0 * ld_dst + r0 + lane;
        if ((r0 + 32 <= rows) && (c0 + 32 <= cols)) {
#pragma unroll
            for (int c = 0; c < 32; ++c) {
                const uint32_t pc = phys_col<L>(lane, c, sh_lane);
                out[c * ld_dst] = ((uint64_t)myhi[pc] << 32) | mylo[pc];
            }
        } else {
            const bool rok = r0 + lane < rows;
            const int64_t cmax = cols - c0;
#pragma unroll 4
            for (int c = 0; c < 32; ++c) {
                if (rok && c < cmax) {
                    const uint32_t pc = phys_col<L>(lane, c, sh_lane);
                    out[c * ld_dst] = ((uint64_t)myhi[pc] << 32) | mylo[pc];
                }
            }
        }
        __syncwarp();
    }
}

// ------------------------------------------------------------------ launchers
template <typename K>
static int grid_for(K kernel, int threads, int64_t ntiles, int warps_per_cta) {
    int dev = 0, sms = 148, occ = 1;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kernel, threads, 0);
    if (occ < 1) occ = 1;
    const int64_t want = (ntiles + warps_per_cta - 1) / warps_per_cta;
    const int64_t cap = (int64_t)sms * occ;
    return (int)(want < cap ? want : cap);
}

TransposeTuning default_tuning(uint32_t elem_bytes) {
    TransposeTuning t;
    t.group = elem_bytes == 4 ? kDefaultGroup32 : kDefaultGroup64;
    t.minb = elem_bytes == 4 ? kDefaultMinB32 : kDefaultMinB64;
    return t;
}

template <int L, bool VEC, int MINB>
static cudaError_t launch_b32(const void *src, void *dst, int64_t rows, int64_t cols, int64_t ld_src,
                              int64_t ld_dst, uint64_t seed, uint32_t group, cudaStream_t st) {
    const uint32_t tiles_r = (uint32_t)((rows + 31) / 32), tiles_c = (uint32_t)((cols + 31) / 32);
    const uint32_t ntiles = tiles_r * tiles_c;
    auto k = transpose_b32_kernel<L, VEC, MINB>;
    const int grid = grid_for(k, kWarps32 * 32, ntiles, kWarps32);
    k<<<grid, kWarps32 * 32, 0, st>>>((const uint32_t *)src, (uint32_t *)dst, rows, cols, ld_src,
                                      ld_dst, seed, tiles_r, tiles_c, ntiles, group);
    return cudaGetLastError();
}

template <int L, bool VEC, int MINB>
static cudaError_t launch_b64(const void *src, void *dst, int64_t rows, int64_t cols, int64_t ld_src,
                              int64_t ld_dst, uint64_t seed, uint32_t group, cudaStream_t st) {
    const uint32_t tiles_r = (uint32_t)((rows + 31) / 32), tiles_c = (uint32_t)((cols + 31) / 32);
    const uint32_t ntiles = tiles_r * tiles_c;
    auto k = transpose_b64_kernel<L, VEC, MINB>;
    const int grid = grid_for(k, kWarps64 * 32, ntiles, kWarps64);
    k<<<grid, kWarps64 * 32, 0, st>>>((const uint64_t *)src, (uint64_t *)dst, rows, cols, ld_src,
                                      ld_dst, seed, tiles_r, tiles_c, ntiles, group);
    return cudaGetLastError();
}

template <int L, bool VEC>
static cudaError_t launch_minb(const void *src, void *dst, int64_t rows, int64_t cols, int64_t ld_src,
                               int64_t ld_dst, uint32_t eb, uint64_t seed, const TransposeTuning &tu,
                               cudaStream_t st) {
    if (eb == 4) {
        switch (tu.minb) {
        case 1: return launch_b32<L, VEC, 1>(src, dst, rows, cols, ld_src, ld_dst, seed, tu.group, st);
        case 3: return launch_b32<L, VEC, 3>(src, dst, rows, cols, ld_src, ld_dst, seed, tu.group, st);
        case 4: return launch_b32<L, VEC, 4>(src, dst, rows, cols, ld_src, ld_dst, seed, tu.group, st);
        default: return launch_b32<L, VEC, 2>(src, dst, rows, cols, ld_src, ld_dst, seed, tu.group, st);
        }
    }
    switch (tu.minb) {
    case 1: return launch_b64<L, VEC, 1>(src, dst, rows, cols, ld_src, ld_dst, seed, tu.group, st);
    case 3: return launch_b64<L, VEC, 3>(src, dst, rows, cols, ld_src, ld_dst, seed, tu.group, st);
    case 4: return launch_b64<L, VEC, 4>(src, dst, rows, cols, ld_src, ld_dst, seed, tu.group, st);
    default: return launch_b64<L, VEC, 2>(src, dst, rows, cols, ld_src, ld_dst, seed, tu.group, st);
    }
}

template <bool VEC>
static cudaError_t dispatch(const void *src, void *dst, int64_t rows, int64_t cols, int64_t ld_src,
                            int64_t ld_dst, uint32_t eb, int layout, uint64_t seed,
                            const TransposeTuning &tu, cudaStream_t st) {
#define RAPK_CASE(LAY) \
    case LAY: return launch_minb<LAY, VEC>(src, dst, rows, cols, ld_src, ld_dst, eb, seed, tu, st);
    switch (layout) {
        RAPK_CASE(RAP_LAYOUT_RAW)
        RAPK_CASE(RAP_LAYOUT_PAD)
        RAPK_CASE(RAP_LAYOUT_XOR)
        RAPK_CASE(RAP_LAYOUT_RAS)
        RAPK_CASE(RAP_LAYOUT_RAP)
    }
#undef RAPK_CASE
    return cudaErrorInvalidValue;
}

cudaError_t launch_transpose_tuned(const void *src, void *dst, int64_t rows, int64_t cols, int64_t ld_src,
                                   int64_t ld_dst, uint32_t elem_bytes, int layout, uint64_t seed,
                                   const TransposeTuning &tu, cudaStream_t st) {
    const bool vec = ((uintptr_t)src % 16 == 0) && ((ld_src * elem_bytes) % 16 == 0);
    return vec ? dispatch<true>(src, dst, rows, cols, ld_src, ld_dst, elem_bytes, layout, seed, tu, st)
               : dispatch<false>(src, dst, rows, cols, ld_src, ld_dst, elem_bytes, layout, seed, tu, st);
}

cudaError_t launch_transpose(const void *src, void *dst, int64_t rows, int64_t cols, int64_t ld_src,
                             int64_t ld_dst, uint32_t elem_bytes, int layout, uint64_t seed,
                             cudaStream_t st) {
    return launch_transpose_tuned(src, dst, rows, cols, ld_src, ld_dst, elem_bytes, layout, seed,
                                  default_tuning(elem_bytes), st);
}

}  // namespace rapk
