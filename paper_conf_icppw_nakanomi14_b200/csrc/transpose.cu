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

#include <atomic>

#include "rap_rng.cuh"
#include "rap_internal.h"

namespace rapk {

// Shared-memory geometry of one warp's 32 x 32 tile, in 4-byte words.
//   RP   : row pitch.  RAP / RAS rows are 64 words wide: element (i, j) sits at word
//          i*64 + j + sh[i] -- the rotation is NOT wrapped in the address, the bank decoder
//          (address mod 32) performs the "mod w" of the paper, so bank(i, j) = (j + P[i]) mod 32
//          exactly as in P:L1005-1016 while every access is base + immediate.
//          RAW / XOR: 32 words; PAD: 33 words (the [32][33] baseline).
//   EW   : 4-byte words per element (1: 32-bit, 2: 64-bit split into lo / hi planes, each a
//          full 32 x RP array, so both planes see the 32-bit bank function).
template <int L>
struct Geom {
    static constexpr int RP = (L == RAP_LAYOUT_RAP || L == RAP_LAYOUT_RAS) ? 64
                            : (L == RAP_LAYOUT_PAD) ? 33 : 32;
};

template <int L, int EW>
__host__ __device__ constexpr int warp_smem_words() { return 32 * Geom<L>::RP * EW; }

// word offset of logical element (row, col) inside a plane; sh = shift of that row
template <int L>
__device__ __forceinline__ uint32_t word_of(uint32_t row, uint32_t col, uint32_t sh) {
    constexpr int RP = Geom<L>::RP;
    if (L == RAP_LAYOUT_XOR) return row * RP + (col ^ row);
    if (L == RAP_LAYOUT_RAS || L == RAP_LAYOUT_RAP) return row * RP + col + sh;
    return row * RP + col;
}

__device__ __forceinline__ uint4 ldg_stream128(const void *p) {
    uint4 r;
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
    return r;
}

// Tile t -> (ti, tj).  Tiles are walked in groups of `group` tile-rows, column by column
// inside a group (group == 0: plain row-major tile order).
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

// Load geometry: a 128-bit load carries NE = 4/EW elements, LPR = 32/NE lanes cover one tile
// row, so one warp instruction loads R = 32/LPR rows and a tile takes G = 32/R instructions.
template <int L, int EW>
struct TileCfg {
    static constexpr int NE = 4 / EW;               // elements per 16-byte chunk
    static constexpr int LPR = 32 / NE;             // lanes per tile row (8 or 16)
    static constexpr int R = 32 / LPR;              // tile rows per load instruction (4 or 2)
    static constexpr int G = 32 / R;                // load instructions per tile (8 or 16)
};

constexpr int kWarpsT = 4;                          // warps per CTA

template <int L, int EW, bool VEC, int DEPTH, int MINB>
__global__ void __launch_bounds__(kWarpsT * 32, MINB)
transpose_kernel(const uint32_t *__restrict__ src, uint32_t *__restrict__ dst, int64_t rows,
                 int64_t cols, int64_t ld_src, int64_t ld_dst, uint64_t seed, uint32_t tiles_r,
                 uint32_t tiles_c, uint32_t ntiles, uint32_t group) {
    using C = TileCfg<L, EW>;
    constexpr int NE = C::NE, R = C::R, G = C::G, LPR = C::LPR;
    constexpr int PW = 32 * Geom<L>::RP;            // plane size in words
    extern __shared__ __align__(16) uint32_t smem_dyn[];
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    uint32_t *tile = smem_dyn + warp * warp_smem_words<L, EW>();

    // ---- T0: the per-warp shift vector, lane i holds sh[i] (P[i] for RAP, r[i] for RAS)
    uint32_t sh_lane = 0;
    if (L == RAP_LAYOUT_RAP) sh_lane = warp_perm<32>(seed, 0, lane, 32);
    if (L == RAP_LAYOUT_RAS) sh_lane = warp_ras_shift(seed, 0, lane, 32);
    // load group g: this lane loads tile row row_g[g], chunk q (elements NE*q .. NE*q+NE-1).
    // RAP: the R rows of group g are P^-1(R*g + 0..R-1) -- one row per residue of P mod R --
    // so each STS of the group hits 32 distinct banks.
    const uint32_t q = lane % LPR, c_in = lane / LPR;
    uint32_t row_g[G], a_g[G];
    uint32_t pinv = lane;
    if (L == RAP_LAYOUT_RAP) {
        tile[sh_lane] = lane;
        __syncwarp();
        pinv = tile[lane];
        __syncwarp();
    }
#pragma unroll
    for (int g = 0; g < G; ++g) {
        const uint32_t rr = (uint32_t)(R * g) + c_in;
        row_g[g] = (L == RAP_LAYOUT_RAP) ? __shfl_sync(kFull, pinv, rr) : rr;
        const uint32_t shg = (L == RAP_LAYOUT_RAP) ? rr : __shfl_sync(kFull, sh_lane, rr);
        a_g[g] = word_of<L>(row_g[g], NE * q, shg);     // first element of the chunk
    }
    const uint32_t drain_base = word_of<L>(lane, 0, sh_lane);

    const uint32_t stride = gridDim.x * kWarpsT;
    uint32_t t = blockIdx.x * kWarpsT + warp;

    auto load = [&](uint4 (&v)[G], uint32_t tt) {
        uint32_t ti, tj;
        tile_coords(tt, tiles_r, tiles_c, group, ti, tj);
        const int64_t r0 = (int64_t)ti * 32, c0 = (int64_t)tj * 32;
        const bool full = (r0 + 32 <= rows) && (c0 + 32 <= cols);
        if (VEC && full) {
            const uint32_t *base = src + (r0 * ld_src + c0 + NE * q) * EW;
#pragma unroll
            for (int g = 0; g < G; ++g) v[g] = ldg_stream128(base + (int64_t)row_g[g] * ld_src * EW);
        } else {
#pragma unroll
            for (int g = 0; g < G; ++g) {
                const int64_t r = r0 + row_g[g];
                const int64_t cc = c0 + NE * q;
                const uint32_t *p = src + (r * ld_src + cc) * EW;
                uint32_t w4[4];
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    const bool ok = (r < rows) && (cc + k / EW < cols);
                    w4[k] = ok ? __ldg(p + k) : 0u;
                }
                v[g] = make_uint4(w4[0], w4[1], w4[2], w4[3]);
            }
        }
    };

    // T1: contiguous (row-wise) write into the RAP tile -- every address is a_g + immediate
    auto store_tile = [&](const uint4 (&v)[G]) {
#pragma unroll
        for (int g = 0; g < G; ++g) {
            const uint32_t w4[4] = {v[g].x, v[g].y, v[g].z, v[g].w};
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                const uint32_t e = k / EW, plane = k % EW;     // element of the chunk, lo/hi word
                uint32_t off;
                if (L == RAP_LAYOUT_XOR) off = word_of<L>(row_g[g], NE * q + e, 0);
                else off = a_g[g] + e;
                tile[plane * PW + off] = w4[k];
            }
        }
    };

    // T2: stride (column-wise) read -- lane i walks its row window -- and coalesced row stores
    auto drain = [&](uint32_t tt) {
        uint32_t ti, tj;
        tile_coords(tt, tiles_r, tiles_c, group, ti, tj);
        const int64_t r0 = (int64_t)ti * 32, c0 = (int64_t)tj * 32;
        const int64_t ostride = ld_dst * EW;                       // words between output rows
        uint32_t *o = dst + (c0 * ld_dst + r0 + lane) * EW;        // this lane's column
        if ((r0 + 32 <= rows) && (c0 + 32 <= cols)) {
#pragma unroll
            for (int c = 0; c < 32; ++c) {
                const uint32_t off = (L == RAP_LAYOUT_XOR) ? word_of<L>(lane, c, 0) : drain_base + c;
                if (EW == 1) *o = tile[off];
                else *reinterpret_cast<uint2 *>(o) = make_uint2(tile[off], tile[PW + off]);
                o += ostride;
            }
        } else {
            const bool rok = r0 + lane < rows;
            const int cmax = (int)min((int64_t)32, cols - c0);
            for (int c = 0; c < cmax; ++c) {
                const uint32_t off = (L == RAP_LAYOUT_XOR) ? word_of<L>(lane, c, 0) : drain_base + c;
                if (rok) {
                    if (EW == 1) *o = tile[off];
                    else *reinterpret_cast<uint2 *>(o) = make_uint2(tile[off], tile[PW + off]);
                }
                o += ostride;
            }
        }
    };

    if (DEPTH == 1) {
        uint4 v[G];
        if (t < ntiles) load(v, t);
        while (t < ntiles) {
            store_tile(v);
            __syncwarp();
            const uint32_t cur = t;
            t += stride;
            if (t < ntiles) load(v, t);                  // T3: next tile in flight
            drain(cur);
            __syncwarp();
        }
    } else {
        uint4 va[G], vb[G];
        if (t < ntiles) load(va, t);
        if (t + stride < ntiles) load(vb, t + stride);
        while (t < ntiles) {
            store_tile(va);
            __syncwarp();
            if (t + 2 * stride < ntiles) load(va, t + 2 * stride);
            drain(t);
            __syncwarp();
            t += stride;
            if (t >= ntiles) break;
            store_tile(vb);
            __syncwarp();
            if (t + 2 * stride < ntiles) load(vb, t + 2 * stride);
            drain(t);
            __syncwarp();
            t += stride;
        }
    }
}

// ------------------------------------------------------------------ launchers
// Host-side launch shape, cached per kernel instantiation and device: the dynamic-smem
// attribute and the occupancy query run once, so a launch costs one cudaGetDevice + one launch.
struct ShapeCache {
    std::atomic<int> occ[kMaxDevices];      // 0 = not yet known
    std::atomic<int> sms[kMaxDevices];
};

template <typename K>
static cudaError_t grid_for(K kernel, ShapeCache &cache, int threads, size_t smem, int64_t ntiles,
                            int warps_per_cta, int ctas_per_sm, int *grid_out) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    if (dev < 0 || dev >= kMaxDevices) return cudaErrorInvalidDevice;
    int occ = cache.occ[dev].load(std::memory_order_relaxed);
    int sms = cache.sms[dev].load(std::memory_order_relaxed);
    if (occ == 0) {
        e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        if (e != cudaSuccess) return e;
        e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kernel, threads, smem);
        if (e != cudaSuccess) return e;
        if (occ < 1) occ = 1;
        cache.sms[dev].store(sms, std::memory_order_relaxed);
        cache.occ[dev].store(occ, std::memory_order_relaxed);
    }
    if (ctas_per_sm > 0 && ctas_per_sm < occ) occ = ctas_per_sm;
    const int64_t want = (ntiles + warps_per_cta - 1) / warps_per_cta;
    const int64_t cap = (int64_t)sms * occ;
    *grid_out = (int)(want < cap ? want : cap);
    return cudaSuccess;
}

TransposeTuning default_tuning(uint32_t elem_bytes) {
    TransposeTuning t;
    t.group = elem_bytes == 4 ? kDefaultGroup32 : kDefaultGroup64;
    t.minb = elem_bytes == 4 ? kDefaultMinB32 : kDefaultMinB64;
    t.depth = elem_bytes == 4 ? kDefaultDepth32 : kDefaultDepth64;
    t.ctas_per_sm = elem_bytes == 4 ? kDefaultCtas32 : kDefaultCtas64;
    return t;
}

template <int L, int EW, bool VEC, int DEPTH, int MINB>
static cudaError_t launch_one(const void *src, void *dst, int64_t rows, int64_t cols, int64_t ld_src,
                              int64_t ld_dst, uint64_t seed, const TransposeTuning &tu, cudaStream_t st) {
    const uint32_t tiles_r = (uint32_t)((rows + 31) / 32), tiles_c = (uint32_t)((cols + 31) / 32);
    const uint32_t ntiles = tiles_r * tiles_c;
    auto k = transpose_kernel<L, EW, VEC, DEPTH, MINB>;
    static ShapeCache cache;
    const size_t smem = sizeof(uint32_t) * warp_smem_words<L, EW>() * kWarpsT;
    int grid = 0;
    const cudaError_t e = grid_for(k, cache, kWarpsT * 32, smem, ntiles, kWarpsT, tu.ctas_per_sm, &grid);
    if (e != cudaSuccess) return e;
    k<<<grid, kWarpsT * 32, smem, st>>>((const uint32_t *)src, (uint32_t *)dst, rows, cols, ld_src,
                                        ld_dst, seed, tiles_r, tiles_c, ntiles, tu.group);
    return cudaGetLastError();
}

template <int L, int EW, bool VEC>
static cudaError_t launch_shape(const void *src, void *dst, int64_t rows, int64_t cols, int64_t ld_src,
                                int64_t ld_dst, uint64_t seed, const TransposeTuning &tu, cudaStream_t st) {
#define RAPK_SHAPE(D, M)                                                                             \
    if (tu.depth == D && tu.minb == M)                                                               \
        return launch_one<L, EW, VEC, D, M>(src, dst, rows, cols, ld_src, ld_dst, seed, tu, st);
#ifdef RAP_TUNING_SWEEP
    RAPK_SHAPE(1, 2) RAPK_SHAPE(1, 3) RAPK_SHAPE(1, 4) RAPK_SHAPE(1, 6) RAPK_SHAPE(1, 8)
    RAPK_SHAPE(2, 2) RAPK_SHAPE(2, 3) RAPK_SHAPE(2, 4) RAPK_SHAPE(2, 6)
#endif
#undef RAPK_SHAPE
    (void)tu;
    return launch_one<L, EW, VEC, EW == 1 ? kDefaultDepth32 : kDefaultDepth64,
                      EW == 1 ? kDefaultMinB32 : kDefaultMinB64>(src, dst, rows, cols, ld_src, ld_dst,
                                                                 seed, tu, st);
}

template <bool VEC>
static cudaError_t dispatch(const void *src, void *dst, int64_t rows, int64_t cols, int64_t ld_src,
                            int64_t ld_dst, uint32_t eb, int layout, uint64_t seed,
                            const TransposeTuning &tu, cudaStream_t st) {
#define RAPK_CASE(LAY)                                                                             \
    case LAY:                                                                                      \
        return eb == 4 ? launch_shape<LAY, 1, VEC>(src, dst, rows, cols, ld_src, ld_dst, seed, tu, st) \
                       : launch_shape<LAY, 2, VEC>(src, dst, rows, cols, ld_src, ld_dst, seed, tu, st);
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
