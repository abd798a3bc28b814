// transpose64.cu -- T1-T3 for 64-bit elements (BASELINE cfg4, 16384^2 float64): the tile holds
// ONE 8-byte element per slot, i.e. the paper's own setting -- "a w x w matrix of double
// (64-bit) numbers", one number per bank word (§III, L1515-1526 §VI) --
// with RAP's map a[i][j] -> a[i][(j + P[i]) mod 32], P = perm(seed, 0, 32) (§IV).
//
// B200 banks are 4 bytes wide, so a double spans a PAIR of banks and a warp's 64-bit shared
// access (256 B) is served in two half-warp wavefronts of 16 doubles each; a half-warp is
// conflict-free when its 16 doubles lie in 16 distinct bank pairs, i.e. distinct column
// residues mod 16 (the double-column index mod 16 names the bank pair).  Under the w = 32 map a
// column read by lanes i = 0..15 hits (c + P[i]) mod 16, which repeats whenever P[i] - P[i'] =
// +-16.  The layout is not changed to avoid it (that is RAP-16, transpose_rap16.cu); instead the
// kernel chooses WHICH lane touches which row (the layout fixes where an element lives, the
// program chooses which thread reads it -- DESIGN reading xv):
//   drain (T2, the DMM stride read): lane l reads row rho(l) = P^-1(l).  Its double of column c
//          sits at rho*64 + c + P[rho] = rho*64 + c + l, so half-warp h hits bank pairs
//          (c + l) mod 16, l = 16h..16h+15: 16 distinct -> the ideal 2 wavefronts per LDS.64.
//          Lane l then stores output element (c, r0 + rho(l)): a permutation of the lanes of one
//          256-byte output row segment, the same 8 sectors as an in-order store.
//   load  (T1, the contiguous write): a 128-bit LDG carries 2 doubles (chunk q = doubles 2q,
//          2q+1); one warp instruction covers 2 rows a = P^-1(2g), b = P^-1(2g+1) -- P[a] even,
//          P[b] odd -- with half-warp h taking chunks q = 8h..8h+7 of both rows.  The two STS.64
//          of a chunk (e = 0, 1) put double 2q+e at bank pair (2q + e + P[row]) mod 16: row a
//          fills the 8 pairs of parity e, row b the 8 of parity 1-e -> 16 distinct per half-warp.
// So every shared-memory request of the RAP tile takes the minimum 2 wavefronts, with the paper's
// w = 32 map, and a tile costs 16 LDG.128 + 32 STS.64 + 32 LDS.64 + 32 STG.64 (112 memory
// instructions; the two-plane kernel of transpose.cu needs 176, RAP-16 128).  Layout RAP64.
// The same kernel serves RAW / PAD ([32][33]) / XOR ([i][j ^ i]) / RAS on 8-byte slots as the
// baselines (rows in natural order, lane l drains row l).
//
// Unwrapped row windows (as transpose.cu): RAP / RAS rows are 64 doubles wide and element (i, j)
// sits at double i*64 + j + sh[i]; the bank decoder performs the "mod 32" (mod 16 bank pairs),
// so every access is base + immediate.
//
// Schedule (as the 32-bit kernel): one warp owns one tile buffer (16 KiB); a CTA of SR warps
// stacked along the input rows drains in lockstep behind one barrier (each output row receives
// SR * 256 B together); persistent CTAs stride over super-tiles; the next tile's loads are in
// flight during the drain.
#include <cuda_runtime.h>
#include <stdint.h>

#include <type_traits>

#include "rap_internal.h"
#include "rap_rng.cuh"

namespace rapk {

template <int L>
struct Geom64 {   // row pitch in doubles
    static constexpr int RP = (L == RAP_LAYOUT_RAP || L == RAP_LAYOUT_RAS) ? 64 : (L == RAP_LAYOUT_PAD) ? 33 : 32;
};

// double offset of logical element (row, col); sh = shift of that row (RAS / RAP)
template <int L>
__device__ __forceinline__ uint32_t slot64(uint32_t row, uint32_t col, uint32_t sh) {
    constexpr uint32_t RP = Geom64<L>::RP;
    if (L == RAP_LAYOUT_XOR) return row * RP + (col ^ row);
    if (L == RAP_LAYOUT_RAS || L == RAP_LAYOUT_RAP) return row * RP + col + sh;
    return row * RP + col;
}

// RAP64_LDG_NA = 1: the loads carry L1::no_allocate; 0 (default): plain read-only loads
// (LDG.E.64 / .128 .CONSTANT), measured faster on cfg4 (profiles/r02_ab64.txt)
#ifndef RAP64_LDG_NA
#define RAP64_LDG_NA 0
#endif
__device__ __forceinline__ uint4 ldg_nc_v4(const void *p) {
#if RAP64_LDG_NA
    uint4 r;
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
    return r;
#else
    return __ldg(reinterpret_cast<const uint4 *>(p));
#endif
}

__device__ __forceinline__ uint2 ldg_nc_v2(const void *p) {
#if RAP64_LDG_NA
    uint2 r;
    asm volatile("ld.global.nc.L1::no_allocate.v2.u32 {%0,%1}, [%2];" : "=r"(r.x), "=r"(r.y) : "l"(p));
    return r;
#else
    return __ldg(reinterpret_cast<const uint2 *>(p));
#endif
}

// ROWS = true: T1 with one LDG.64 per tile row (lane j reads double j, 256 B per instruction,
// 32 per tile) and one STS.64 per row: lanes j = 0..15 of row i hit bank pairs (j + P[i]) mod 16,
// distinct for any P -- the row write needs no grouping.  ROWS = false: the LDG.128 grouping above.
// P32 (tuning, RAP32_PAIR): the same kernel moves a 32-bit matrix as a matrix of virtual 8-byte
// elements v(i, k) = (a[i][2k], a[i][2k+1]) -- column pairs, so `cols` / `ld_src` count pairs and
// `ld_dst` counts 32-bit words.  A tile is 32 rows x 64 words (256-byte input rows, one LDG.64
// per row); the drain's slot (rho, c) holds output elements (2c, rho) and (2c+1, rho), stored by
// two STG.32 into two 128-byte output row segments.
template <int L, bool VEC, int SR, int MINB, bool ROWS, bool P32 = false>
__global__ void __launch_bounds__(SR * 32, MINB)
transpose64_kernel(const uint2 *__restrict__ src, uint2 *__restrict__ dst, int64_t rows, int64_t cols,
                   int64_t ld_src, int64_t ld_dst, const TileShifts ts, uint32_t tiles_r, uint32_t tiles_c) {
    constexpr int RP = Geom64<L>::RP;
    constexpr bool RAP = (L == RAP_LAYOUT_RAP);
    extern __shared__ __align__(16) uint2 smem64[];
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    uint2 *tile = smem64 + warp * (32 * RP);

    // T0 (host, tile_shifts): P / P^-1 (RAP) or r (RAS) of the launch
    const uint32_t sh_lane = (RAP || L == RAP_LAYOUT_RAS) ? shift_byte(ts.sh, lane) : 0u;
    const uint32_t inv_lane = RAP ? shift_byte(ts.inv, lane) : lane;

    // T1 lane geometry: half-warp h = lane / 16 takes chunks q = 8h .. 8h+7 of both rows of a
    // group; rsel picks the row (RAP: a = P^-1(2g) with P even, b = P^-1(2g+1) with P odd)
    const uint32_t rsel = (lane >> 3) & 1u;
    const uint32_t q = ((lane >> 4) << 3) | (lane & 7u);
    constexpr int NG = ROWS ? 1 : 16;                   // (ROWS: unused)
    uint32_t row_g[NG], a_g[NG];
#pragma unroll
    for (int g = 0; g < NG; ++g) {
        const uint32_t rr = 2u * g + rsel;
        row_g[g] = RAP ? __shfl_sync(kFull, inv_lane, rr) : rr;
        const uint32_t shg = RAP ? rr : (L == RAP_LAYOUT_RAS ? __shfl_sync(kFull, sh_lane, rr) : 0u);
        a_g[g] = slot64<L>(row_g[g], 2u * q, shg);          // double 2q; double 2q+1 follows
    }
    // ROWS: lane j writes double j of row r at st_off[r] (RAS / RAP: r*RP + j + sh[r])
    constexpr int NR = ROWS ? 32 : 1;
    uint32_t st_off[NR];
#pragma unroll
    for (int r = 0; r < NR; ++r) {
        // sh[r] read straight from the kernel parameter (r is a compile-time constant): a
        // warp-uniform value, so the row base r*RP + sh[r] can live in a uniform register
        const uint32_t shr = (RAP || L == RAP_LAYOUT_RAS) ? (ts.sh[r >> 2] >> (8 * (r & 3))) & 0xffu : 0u;
        st_off[r] = slot64<L>((uint32_t)r, lane, shr);
    }
    // T2 lane geometry: lane l drains row rho = P^-1(l) (RAP) or l; column c at drain_base + c
    // (RAP64_NATURAL_DRAIN: lane l drains row l under RAP too -- an ablation with ~2-way
    // conflicted LDS.64, to measure what the permuted output lanes cost)
#ifdef RAP64_NATURAL_DRAIN
    const uint32_t rho = lane;
    const uint32_t drain_base = slot64<L>(lane, 0, sh_lane);
#else
    const uint32_t rho = inv_lane;
    const uint32_t drain_base = RAP ? rho * RP + lane : slot64<L>(lane, 0, sh_lane);
#endif

    const uint32_t nst = ((tiles_r + SR - 1) / SR) * tiles_c;
    auto coords = [&](uint32_t st, uint32_t &ti, uint32_t &tj) -> bool {
        const uint32_t si = st / tiles_c;
        tj = st - si * tiles_c;
        ti = si * SR + warp;
        return ti < tiles_r;
    };

    using Buf = typename std::conditional<ROWS, uint2[32], uint4[16]>::type;
    auto load_rows = [&](uint2 (&v)[32], uint32_t ti, uint32_t tj) {
        const int64_t r0 = (int64_t)ti * 32, c0 = (int64_t)tj * 32;
        const uint2 *p = src + r0 * ld_src + c0 + lane;
        if (r0 + 32 <= rows && c0 + 32 <= cols) {
#pragma unroll
            for (int r = 0; r < 32; ++r) v[r] = ldg_nc_v2(p + (int64_t)r * ld_src);
        } else {
            const bool cok = c0 + lane < cols;
#pragma unroll
            for (int r = 0; r < 32; ++r)
                v[r] = (cok && r0 + r < rows) ? __ldg(p + (int64_t)r * ld_src) : make_uint2(0u, 0u);
        }
    };
    auto store_rows = [&](const uint2 (&v)[32]) {
#pragma unroll
        for (int r = 0; r < 32; ++r) tile[st_off[r]] = v[r];
    };
    auto load_groups = [&](uint4 (&v)[16], uint32_t ti, uint32_t tj) {
        const int64_t r0 = (int64_t)ti * 32, c0 = (int64_t)tj * 32;
        if (VEC && r0 + 32 <= rows && c0 + 32 <= cols) {
            const uint2 *base = src + r0 * ld_src + c0 + 2 * q;
#pragma unroll
            for (int g = 0; g < 16; ++g) v[g] = ldg_nc_v4(base + (int64_t)row_g[g] * ld_src);
        } else {
#pragma unroll
            for (int g = 0; g < 16; ++g) {
                const int64_t r = r0 + row_g[g], c = c0 + 2 * q;
                const uint2 *p = src + r * ld_src + c;
                const uint2 x0 = (r < rows && c < cols) ? __ldg(p) : make_uint2(0u, 0u);
                const uint2 x1 = (r < rows && c + 1 < cols) ? __ldg(p + 1) : make_uint2(0u, 0u);
                v[g] = make_uint4(x0.x, x0.y, x1.x, x1.y);
            }
        }
    };

    // T1: the contiguous write into the tile, two STS.64 per chunk
    auto store_groups = [&](const uint4 (&v)[16]) {
#pragma unroll
        for (int g = 0; g < 16; ++g) {
            if (L == RAP_LAYOUT_XOR) {
                tile[a_g[g]] = make_uint2(v[g].x, v[g].y);
                tile[a_g[g] ^ 1u] = make_uint2(v[g].z, v[g].w);   // (2q+1) ^ row = (2q ^ row) ^ 1
            } else {
                tile[a_g[g]] = make_uint2(v[g].x, v[g].y);
                tile[a_g[g] + 1] = make_uint2(v[g].z, v[g].w);
            }
        }
    };

    // T2: the stride (column) read and 256-byte output rows
    auto drain = [&](uint32_t ti, uint32_t tj) {
        const int64_t r0 = (int64_t)ti * 32, c0 = (int64_t)tj * 32;
        if constexpr (P32) {
            uint32_t *o = reinterpret_cast<uint32_t *>(dst) + 2 * c0 * ld_dst + r0 + rho;
            const bool rok = r0 + rho < rows;
            const int cmax = (int)min((int64_t)32, cols - c0);
            if (r0 + 32 <= rows && cmax == 32) {
#pragma unroll
                for (int c = 0; c < 32; ++c) {
                    const uint32_t off = (L == RAP_LAYOUT_XOR) ? drain_base ^ (uint32_t)c : drain_base + c;
                    const uint2 x = tile[off];
                    o[0] = x.x;
                    o[ld_dst] = x.y;
                    o += 2 * ld_dst;
                }
            } else {
                for (int c = 0; c < cmax; ++c) {
                    const uint32_t off = (L == RAP_LAYOUT_XOR) ? drain_base ^ (uint32_t)c : drain_base + c;
                    if (rok) {
                        const uint2 x = tile[off];
                        o[0] = x.x;
                        o[ld_dst] = x.y;
                    }
                    o += 2 * ld_dst;
                }
            }
            return;
        }
        uint2 *o = dst + c0 * ld_dst + r0 + rho;
        if (r0 + 32 <= rows && c0 + 32 <= cols) {
#pragma unroll
            for (int c = 0; c < 32; ++c) {
                const uint32_t off = (L == RAP_LAYOUT_XOR) ? drain_base ^ (uint32_t)c
                                                           : drain_base + c;
                *o = tile[off];
                o += ld_dst;
            }
        } else {
            const bool rok = r0 + rho < rows;
            const int cmax = (int)min((int64_t)32, cols - c0);
            for (int c = 0; c < cmax; ++c) {
                const uint32_t off = (L == RAP_LAYOUT_XOR) ? drain_base ^ (uint32_t)c
                                                           : drain_base + c;
                if (rok) *o = tile[off];
                o += ld_dst;
            }
        }
    };

    auto load = [&](Buf &v, uint32_t ti, uint32_t tj) {
        if constexpr (ROWS) load_rows(v, ti, tj); else load_groups(v, ti, tj);
    };
    auto store_tile = [&](const Buf &v) {
        if constexpr (ROWS) store_rows(v); else store_groups(v);
    };

    uint32_t st = blockIdx.x, ti = 0, tj = 0;
    bool act = st < nst && coords(st, ti, tj);
    Buf v;
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

// CTA shape: SR warps stacked along the input rows (measured for 64-bit tiles in round 1:
// 12 x 1 with one CTA per SM, profiles/r01_tune_transpose*.txt); RAP64_SR overrides for tuning
#ifndef RAP64_SR
#define RAP64_SR 12
#endif
#ifndef RAP64_MINB
#define RAP64_MINB 1
#endif
#ifndef RAP64_ROWS
#define RAP64_ROWS 1
#endif

template <int L, bool VEC, int SR, int MINB, bool ROWS = RAP64_ROWS, bool P32 = false>
static cudaError_t launch64_one(const void *src, void *dst, int64_t rows, int64_t cols, int64_t ld_src,
                                int64_t ld_dst, uint64_t seed, cudaStream_t st) {
    auto k = transpose64_kernel<L, VEC, SR, MINB, ROWS, P32>;
    static ShapeCache cache;
    const size_t smem = sizeof(uint2) * 32 * Geom64<L>::RP * SR;
    const uint32_t tiles_r = (uint32_t)((rows + 31) / 32), tiles_c = (uint32_t)((cols + 31) / 32);
    const int64_t nst = (int64_t)((tiles_r + SR - 1) / SR) * tiles_c;
    int grid = 0;
#ifdef RAP64_CARVEOUT
    static bool carve = [&] {
        return cudaFuncSetAttribute(k, cudaFuncAttributePreferredSharedMemoryCarveout, RAP64_CARVEOUT) == cudaSuccess;
    }();
    (void)carve;
#endif
    const cudaError_t e = cached_grid(k, cache, SR * 32, smem, nst, 0, &grid);
    if (e != cudaSuccess) return e;
    TileShifts ts = tile_shifts(L, seed);
    if (P32) pdl_forget(st);
    else ts.early = pdl_early_loads(st, src, rows, cols, ld_src, dst, cols, rows, ld_dst, 8u) ? 1u : 0u;
    return launch_ex(k, grid, SR * 32, smem, st, 1, (const uint2 *)src, (uint2 *)dst, rows, cols, ld_src, ld_dst, ts,
                     tiles_r, tiles_c);
}

template <int L, bool VEC>
static cudaError_t launch64_layout(const void *src, void *dst, int64_t rows, int64_t cols, int64_t ld_src,
                                   int64_t ld_dst, uint64_t seed, cudaStream_t st) {
    // a handful of tiles (a 32 x 32 problem): one single-warp CTA per tile
    if (((rows + 31) / 32) * ((cols + 31) / 32) <= kSmallTiles)
        return launch64_one<L, VEC, 1, 1>(src, dst, rows, cols, ld_src, ld_dst, seed, st);
    return launch64_one<L, VEC, RAP64_SR, RAP64_MINB>(src, dst, rows, cols, ld_src, ld_dst, seed, st);
}

cudaError_t launch_transpose64(const void *src, void *dst, int64_t rows, int64_t cols, int64_t ld_src,
                               int64_t ld_dst, int layout, uint64_t seed, cudaStream_t st) {
    const bool vec = ((uintptr_t)src % 16 == 0) && (ld_src % 2 == 0);
#define RAPK64_CASE(LAY)                                                                             \
    case LAY:                                                                                        \
        return vec ? launch64_layout<LAY, true>(src, dst, rows, cols, ld_src, ld_dst, seed, st)      \
                   : launch64_layout<LAY, false>(src, dst, rows, cols, ld_src, ld_dst, seed, st);
    switch (layout) {
        RAPK64_CASE(RAP_LAYOUT_RAW)
        RAPK64_CASE(RAP_LAYOUT_PAD)
        RAPK64_CASE(RAP_LAYOUT_XOR)
        RAPK64_CASE(RAP_LAYOUT_RAS)
        RAPK64_CASE(RAP_LAYOUT_RAP)
    }
#undef RAPK64_CASE
    return cudaErrorInvalidValue;
}

#ifndef RAP32_PAIR_SR
#define RAP32_PAIR_SR 12
#endif
#ifndef RAP32_PAIR_MINB
#define RAP32_PAIR_MINB 1
#endif
// 32-bit transposes through column-pair 8-byte slots (RAP32_PAIR tuning path of transpose.cu):
// requires an even `cols`, an even `ld_src` and an 8-byte aligned source (the caller checks)
cudaError_t launch_transpose_pair32(const void *src, void *dst, int64_t rows, int64_t cols, int64_t ld_src,
                                    int64_t ld_dst, int layout, uint64_t seed, cudaStream_t st) {
#define RAPK32P_CASE(LAY)                                                                            \
    case LAY:                                                                                        \
        return launch64_one<LAY, true, RAP32_PAIR_SR, RAP32_PAIR_MINB, true, true>(src, dst, rows, cols / 2, \
                                                                               ld_src / 2, ld_dst, seed, st);
    switch (layout) {
        RAPK32P_CASE(RAP_LAYOUT_RAW)
        RAPK32P_CASE(RAP_LAYOUT_PAD)
        RAPK32P_CASE(RAP_LAYOUT_XOR)
        RAPK32P_CASE(RAP_LAYOUT_RAS)
        RAPK32P_CASE(RAP_LAYOUT_RAP)
    }
#undef RAPK32P_CASE
    return cudaErrorInvalidValue;
}

}  // namespace rapk
