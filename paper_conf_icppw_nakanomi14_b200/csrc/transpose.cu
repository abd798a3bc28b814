// transpose.cu -- steps T0-T3 of the RAP hot path: the out-of-place HBM transpose staged
// through 32 x 32 shared-memory tiles laid out RAW / PAD / XOR / RAS / RAP.
//
// Paper: the RAP CRSW transpose of one 32 x 32 tile (§VI) moves a[i][j] to
// b[j][i] with a[i][j] stored at a[i][(j + P[i]) mod 32] (§IV), so that the
// row-wise (contiguous) write AND the column-wise (stride) read of the tile are both
// conflict-free for every P (Theorem 2).
//
// B200 design: one warp owns one 32 x 32 tile buffer (only __syncwarp inside a
// tile); a CTA of SR x SC warps works on an SR x SC block of tiles and drains it in lockstep
// (one CTA barrier per super-tile); persistent CTAs stride over super-tiles, and the next
// tile's global loads are in flight while the current tile is drained.
//   load  : 128-bit LDG.  One warp instruction covers 4 tile rows x 128 B.  Under RAP the 4
//           rows are chosen as P^-1(4g+0..3), i.e. rows whose P values cover the 4 residues
//           mod 4, which makes each of the 4 following STS.32 hit 32 distinct banks:
//           bank(row, 4q+k) = (4q + k + 4g + c) mod 32 is injective in (c, q).
//   smem  : STS.32 of element (i, j) at word i*64 + j + P[i] (unwrapped RAP row window, Geom).
//   drain : lane i reads column c of the tile at word i*64 + P[i] + c: the DMM stride access,
//           banks (c + P[i]) mod 32 distinct because P is a permutation; then 128-byte
//           coalesced STG.32 of output row c (or a staging tile + TMA store, TMAS).
// 64-bit elements: 32 banks of 4 bytes (the paper assumed one double per bank word,
// P:L278-283, L860), so a tile of doubles is split into two 32-bit RAP planes (low / high
// words) with identical addressing; every smem access stays a 32-lane 4-byte access.  (The
// other encodings: one double per 8-byte slot, transpose64.cu / RAP_LAYOUT_RAP64; RAP over 16
// double banks, transpose_rap16.cu / RAP_LAYOUT_RAP16.)
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>
#include <cstring>

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
// RAP32_WRAP (tuning, default 0): RAP / RAS rows 32 words wide with the rotation wrapped in the
// address arithmetic, (j + sh[i]) & 31 -- half the shared memory per tile, two more ALU
// operations per shared access
#ifndef RAP32_WRAP
#define RAP32_WRAP 0
#endif
template <int L>
struct Geom {
    static constexpr bool WRAP = RAP32_WRAP && (L == RAP_LAYOUT_RAP || L == RAP_LAYOUT_RAS);
    static constexpr int RP = WRAP ? 32 : (L == RAP_LAYOUT_RAP || L == RAP_LAYOUT_RAS) ? 64
                            : (L == RAP_LAYOUT_PAD) ? 33 : 32;
};

template <int L, int EW>
__host__ __device__ constexpr int warp_smem_words() { return 32 * Geom<L>::RP * EW; }

// word offset of logical element (row, col) inside a plane; sh = shift of that row
template <int L>
__device__ __forceinline__ uint32_t word_of(uint32_t row, uint32_t col, uint32_t sh) {
    constexpr int RP = Geom<L>::RP;
    if (L == RAP_LAYOUT_XOR) return row * RP + (col ^ row);
    if (Geom<L>::WRAP) return row * RP + ((col + sh) & 31u);
    if (L == RAP_LAYOUT_RAS || L == RAP_LAYOUT_RAP) return row * RP + col + sh;
    return row * RP + col;
}

// RAP32_LDG_NA = 1: 128-bit loads with L1::no_allocate; 0 (default): plain read-only loads
// (LDG.E.128.CONSTANT) -- +4-5 % on cfg3 in interleaved A/B runs (profiles/r02_ab32.txt)
#ifndef RAP32_LDG_NA
#define RAP32_LDG_NA 0
#endif
__device__ __forceinline__ uint4 ldg_stream128(const void *p) {
#if RAP32_LDG_NA
    uint4 r;
    // (an L2::256B prefetch hint measured no different, profiles/r01_tune_transpose_tma.txt)
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
    return r;
#else
    return __ldg(reinterpret_cast<const uint4 *>(p));
#endif
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

// CTA = SR x SC warps working on an SR x SC block of tiles ("super-tile") in lockstep: warp w
// owns tile (w % SR, w / SR) of the block, and a CTA barrier before the drains makes the SC*32
// input rows / SR*32-element output row runs of neighbouring warps reach DRAM together
// (measured: +2-4 % over free-running warps, profiles/r01_tune_transpose.txt).
// TMA store path (TMAS): the drains of a super-tile write a dense (SC*32) x (SR*32) staging
// tile in shared memory (row-contiguous, conflict-free) and one thread stores it to HBM with a
// single cp.async.bulk.tensor (out-of-range rows/columns of edge super-tiles are clipped by TMA).
__device__ __forceinline__ void tma_store_2d(const CUtensorMap *map, const void *smem, int32_t x, int32_t y) {
    const uint32_t s = static_cast<uint32_t>(__cvta_generic_to_shared(smem));
    asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%1, %2}], [%3];"
                 :: "l"(map), "r"(x), "r"(y), "r"(s) : "memory");
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}
__device__ __forceinline__ void tma_wait_read() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
__device__ __forceinline__ void tma_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

// RAP32_KP: 32-bit transposes through the row-pair-plane form (KP above) -- tuning flag, off:
// measured 5.85 against 6.08 TB/s for the default at 8192^2 and 6.05 against 6.16 at 16384^2
// (profiles/r02_ab_kp*.txt), so 256-byte output rows are not what the 32-bit kernel lacks
#ifndef RAP32_KP
#define RAP32_KP 0
#endif
// RAP32_PAIR: 32-bit transposes through column-pair 8-byte slots (transpose64.cu's P32 form) --
// tuning flag, off
#ifndef RAP32_PAIR
#define RAP32_PAIR 0
#endif
#ifndef RAP32_KP_SR
#define RAP32_KP_SR 12
#endif
#ifndef RAP32_KP_MINB
#define RAP32_KP_MINB 1
#endif
#ifndef RAP32_KP_CL
#define RAP32_KP_CL 1
#endif

// Cluster lockstep (CL > 1): the CL CTAs of a thread-block cluster take the CL row blocks of one
// (CL*SR) x SC-tile cluster super-tile and drain behind one barrier.cluster, so each output row
// receives CL*SR*128 B at once (+1.5-2 % over CL = 1, profiles/r01_probe_transpose.txt; 8 CTAs
// +1.5 % over 4, profiles/r02_ab32s3.txt).
__device__ __forceinline__ void cluster_sync_relaxed() {
    asm volatile("barrier.cluster.arrive.relaxed.aligned;" ::: "memory");
    asm volatile("barrier.cluster.wait.aligned;" ::: "memory");
}

// KP (row-pair planes, 32-bit elements): the kernel runs its EW = 2 form on a matrix of virtual
// 8-byte elements v(i, j) = (src[2i][j], src[2i+1][j]): plane 0 of a tile holds input row 2i,
// plane 1 input row 2i+1, both under the tile's RAP map, and the transpose of the virtual matrix
// IS the 32-bit transpose -- output element v(j, i) = (out[j][2i], out[j][2i+1]) is contiguous.
// So a warp moves a 64 x 32 block of 32-bit elements per tile (8 KiB) and the drain writes each
// output row as one 256-byte STG.64 instead of a 128-byte STG.32, like the 64-bit kernel.  Loads:
// one LDG.128 = 4 elements of one input row; instruction g (16 per tile) takes plane g & 1 of the
// 4 virtual rows P^-1(4 (g >> 1) + 0..3) -- one per residue of P mod 4 -- so each STS.32 is
// conflict-free as in the 32-bit kernel.  Here `rows` counts virtual rows (input rows / 2) and
// ld_dst is in 8-byte units; ld_src stays in 32-bit words.
template <int L, int EW, bool VEC, int DEPTH, int MINB, bool VST, int SR, int SC, bool PEERS, bool TMAS,
          int CL = 1, bool KP = false>
__global__ void __launch_bounds__(SR * SC * 32, MINB)
transpose_kernel(const uint32_t *__restrict__ src, uint32_t *__restrict__ dst, int64_t rows,
                 int64_t cols, int64_t ld_src, int64_t ld_dst, const TileShifts ts, uint32_t tiles_r,
                 uint32_t tiles_c, bool vst_ok, PeerOut peers, const __grid_constant__ CUtensorMap tmap) {
    static_assert(!TMAS || (DEPTH == 1 && !PEERS && SR * 32 <= 256), "TMA store: depth 1, box <= 256");
    static_assert(CL == 1 || (DEPTH == 1 && !TMAS), "cluster lockstep: depth 1, no TMA store");
    static_assert(!KP || (EW == 2 && VEC && DEPTH == 1 && !VST && !PEERS && !TMAS), "row-pair planes: EW 2 form");
    using C = TileCfg<L, EW>;
    constexpr int NE = C::NE, R = C::R, G = C::G, LPR = C::LPR;
    constexpr int PW = 32 * Geom<L>::RP;            // plane size in words
    extern __shared__ __align__(16) uint32_t smem_dyn[];
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    uint32_t *tile = smem_dyn + warp * warp_smem_words<L, EW>();
    uint32_t *staging = smem_dyn + SR * SC * warp_smem_words<L, EW>();   // TMAS: (SC*32) x (SR*32) x EW words

    // ---- T0: the shift vector of the launch (computed once on the host, tile_shifts), lane i
    // holds sh[i] (P[i] for RAP, r[i] for RAS)
    uint32_t sh_lane = 0;
    if (L == RAP_LAYOUT_RAP || L == RAP_LAYOUT_RAS) sh_lane = shift_byte(ts.sh, lane);
    // load group g: this lane loads tile row row_g[g], chunk q (elements NE*q .. NE*q+NE-1).
    // RAP: the R rows of group g are P^-1(R*g + 0..R-1) -- one row per residue of P mod R --
    // so each STS of the group hits 32 distinct banks.
    const uint32_t q = lane % LPR, c_in = lane / LPR;
    constexpr bool WRAP = Geom<L>::WRAP;
    uint32_t row_g[G], a_g[G], rot_g[WRAP ? G : 1];
    const uint32_t pinv = (L == RAP_LAYOUT_RAP) ? shift_byte(ts.inv, lane) : lane;
#pragma unroll
    for (int g = 0; g < G; ++g) {
        const uint32_t rr = (uint32_t)(R * g) + c_in;
        row_g[g] = (L == RAP_LAYOUT_RAP) ? __shfl_sync(kFull, pinv, rr) : rr;
        const uint32_t shg = (L == RAP_LAYOUT_RAP) ? rr : __shfl_sync(kFull, sh_lane, rr);
        if constexpr (WRAP) {
            a_g[g] = row_g[g] * Geom<L>::RP;            // row base; column (NE*q + e + sh) & 31
            rot_g[g] = NE * q + shg;
        } else {
            a_g[g] = word_of<L>(row_g[g], NE * q, shg);  // first element of the chunk
        }
    }
    const uint32_t drain_base = word_of<L>(lane, 0, sh_lane);
    if constexpr (KP) {          // row-pair planes: chunk kq of 4 elements, virtual row set kc
        const uint32_t kq = lane & 7u, kc = lane >> 3;
#pragma unroll
        for (int g = 0; g < G; ++g) {
            const uint32_t p = (uint32_t)g & 1u, rr = 4u * (uint32_t)(g >> 1) + kc;
            const uint32_t vr = (L == RAP_LAYOUT_RAP) ? __shfl_sync(kFull, pinv, rr) : rr;
            const uint32_t shv = (L == RAP_LAYOUT_RAP) ? rr
                               : (L == RAP_LAYOUT_RAS) ? __shfl_sync(kFull, sh_lane, rr) : 0u;
            row_g[g] = 2u * vr + p;                               // input row within the 64-row block
            a_g[g] = p * PW + ((L == RAP_LAYOUT_XOR) ? vr * Geom<L>::RP + ((4u * kq) ^ vr)
                                                     : word_of<L>(vr, 4u * kq, shv));
        }
    }

    // super-tile s -> this warp's tile (ti, tj); false when it falls outside the matrix.  With
    // clusters, s counts cluster super-tiles and CTA rank `crank` takes row block crank of it.
    uint32_t crank = 0, st_first = blockIdx.x, st_step = gridDim.x;
    if (CL > 1) {
        asm("mov.u32 %0, %%cluster_ctarank;" : "=r"(crank));
        asm("mov.u32 %0, %%clusterid.x;" : "=r"(st_first));
        asm("mov.u32 %0, %%nclusterid.x;" : "=r"(st_step));
    }
    const uint32_t stc = (tiles_c + SC - 1) / SC;
    const uint32_t nst = ((tiles_r + SR * CL - 1) / (SR * CL)) * stc;
    const uint32_t wr = crank * SR + warp % SR, wc = warp / SR;
    auto coords = [&](uint32_t st, uint32_t &ti, uint32_t &tj) -> bool {
        const uint32_t si = st / stc, sj = st - si * stc;
        ti = si * SR * CL + wr;
        tj = sj * SC + wc;
        return ti < tiles_r && tj < tiles_c;
    };

    auto load = [&](uint4 (&v)[G], uint32_t ti, uint32_t tj) {
        const int64_t r0 = (int64_t)ti * 32, c0 = (int64_t)tj * 32;
        const bool full = (r0 + 32 <= rows) && (c0 + 32 <= cols);
        if constexpr (KP) {
            const uint32_t *base = src + 2 * r0 * ld_src + c0 + 4 * (lane & 7u);
            if (full) {
#pragma unroll
                for (int g = 0; g < G; ++g) v[g] = ldg_stream128(base + (int64_t)row_g[g] * ld_src);
            } else {
                const int64_t prow_end = 2 * rows, cc = c0 + 4 * (lane & 7u);
#pragma unroll
                for (int g = 0; g < G; ++g) {
                    const int64_t r = 2 * r0 + row_g[g];
                    const uint32_t *pp = base + (int64_t)row_g[g] * ld_src;
                    uint32_t w4[4];
#pragma unroll
                    for (int k = 0; k < 4; ++k) w4[k] = (r < prow_end && cc + k < cols) ? __ldg(pp + k) : 0u;
                    v[g] = make_uint4(w4[0], w4[1], w4[2], w4[3]);
                }
            }
        } else if (VEC && full) {
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
        if constexpr (KP) {      // 4 consecutive elements of one input row into its plane
#pragma unroll
            for (int g = 0; g < G; ++g) {
                const uint32_t w4[4] = {v[g].x, v[g].y, v[g].z, v[g].w};
#pragma unroll
                for (int k = 0; k < 4; ++k)
                    tile[(L == RAP_LAYOUT_XOR) ? (a_g[g] ^ (uint32_t)k) : a_g[g] + k] = w4[k];
            }
        } else {
#pragma unroll
            for (int g = 0; g < G; ++g) {
                const uint32_t w4[4] = {v[g].x, v[g].y, v[g].z, v[g].w};
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    const uint32_t e = k / EW, plane = k % EW;     // element of the chunk, lo/hi word
                    uint32_t off;
                    if (L == RAP_LAYOUT_XOR) off = word_of<L>(row_g[g], NE * q + e, 0);
                    else if constexpr (WRAP) off = a_g[g] + ((rot_g[g] + e) & 31u);
                    else off = a_g[g] + e;
                    tile[plane * PW + off] = w4[k];
                }
            }
        }
    };

    // T2: stride (column-wise) read -- lane i walks its row window -- and coalesced row stores
    auto drain = [&](uint32_t ti, uint32_t tj) {
        const int64_t r0 = (int64_t)ti * 32, c0 = (int64_t)tj * 32;
        const int64_t ostride = ld_dst * EW;                       // words between output rows
        // output tile origin: (c0, r0) of dst, or -- fused exchange (NEXT-2) -- of the output
        // shard of rank h = c0 / M, written straight over NVLink through its mapped pointer
        uint32_t *obase = dst;
        int64_t orow = c0, ocol = r0;
        if (PEERS) {
            const int64_t h = c0 / peers.M;
            obase = reinterpret_cast<uint32_t *>(peers.ptr[h]);
            orow = c0 - h * peers.M;
            ocol = peers.col_off + r0;
        }
        uint32_t *o = obase + (orow * ld_dst + ocol + lane) * EW;    // this lane's column
        if (VST && vst_ok && (r0 + 32 <= rows) && (c0 + 32 <= cols)) {
            // 128-bit stores: each lane reads NE consecutive columns of its row, a butterfly of
            // __shfl_xor_sync transposes NE x NE blocks among NE lanes, and lane NE*p + k then
            // holds rows NE*p .. NE*p+NE-1 of column c+k -- one 16-byte chunk of output row c+k.
            const uint32_t k = lane % NE, p = lane / NE;
            uint32_t *ob = obase + ((orow + k) * ld_dst + ocol + NE * p) * EW;
#pragma unroll
            for (int cg = 0; cg < 32 / NE; ++cg) {
                uint32_t r[4];
                if (EW == 1) {
#pragma unroll
                    for (int m = 0; m < 4; ++m) {
                        const uint32_t off = (L == RAP_LAYOUT_XOR || WRAP) ? word_of<L>(lane, 4 * cg + m, sh_lane) : drain_base + 4 * cg + m;
                        r[m] = tile[off];
                    }
                    const bool b0 = lane & 1u, b1 = lane & 2u;
                    uint32_t x = __shfl_xor_sync(kFull, b0 ? r[0] : r[1], 1);
                    if (b0) r[0] = x; else r[1] = x;
                    x = __shfl_xor_sync(kFull, b0 ? r[2] : r[3], 1);
                    if (b0) r[2] = x; else r[3] = x;
                    x = __shfl_xor_sync(kFull, b1 ? r[0] : r[2], 2);
                    if (b1) r[0] = x; else r[2] = x;
                    x = __shfl_xor_sync(kFull, b1 ? r[1] : r[3], 2);
                    if (b1) r[1] = x; else r[3] = x;
                } else {
#pragma unroll
                    for (int m = 0; m < 2; ++m) {
                        const uint32_t off = (L == RAP_LAYOUT_XOR || WRAP) ? word_of<L>(lane, 2 * cg + m, sh_lane) : drain_base + 2 * cg + m;
                        r[2 * m] = tile[off];
                        r[2 * m + 1] = tile[PW + off];
                    }
                    const bool b0 = lane & 1u;
                    const uint32_t xl = __shfl_xor_sync(kFull, b0 ? r[0] : r[2], 1);
                    const uint32_t xh = __shfl_xor_sync(kFull, b0 ? r[1] : r[3], 1);
                    if (b0) { r[0] = xl; r[1] = xh; } else { r[2] = xl; r[3] = xh; }
                }
                *reinterpret_cast<uint4 *>(ob) = make_uint4(r[0], r[1], r[2], r[3]);
                ob += ostride * NE;
            }
        } else if ((r0 + 32 <= rows) && (c0 + 32 <= cols)) {
#pragma unroll
            for (int c = 0; c < 32; ++c) {
                const uint32_t off = (L == RAP_LAYOUT_XOR || WRAP) ? word_of<L>(lane, c, sh_lane) : drain_base + c;
                if (EW == 1) *o = tile[off];
                else *reinterpret_cast<uint2 *>(o) = make_uint2(tile[off], tile[PW + off]);
                o += ostride;
            }
        } else {
            const bool rok = r0 + lane < rows;
            const int cmax = (int)min((int64_t)32, cols - c0);
            for (int c = 0; c < cmax; ++c) {
                const uint32_t off = (L == RAP_LAYOUT_XOR || WRAP) ? word_of<L>(lane, c, sh_lane) : drain_base + c;
                if (rok) {
                    if (EW == 1) *o = tile[off];
                    else *reinterpret_cast<uint2 *>(o) = make_uint2(tile[off], tile[PW + off]);
                }
                o += ostride;
            }
        }
    };

    // TMAS drain: tile (wr, wc) of the super-tile -> staging rows wc*32 + c, columns wr*32 + lane
    auto drain_staging = [&]() {
        constexpr int SW = SR * 32;                                // staging row length (elements)
#pragma unroll
        for (int c = 0; c < 32; ++c) {
            const uint32_t off = (L == RAP_LAYOUT_XOR || WRAP) ? word_of<L>(lane, c, sh_lane) : drain_base + c;
            const uint32_t e = (wc * 32 + c) * SW + wr * 32 + lane;
            if (EW == 1) staging[e] = tile[off];
            else *reinterpret_cast<uint2 *>(staging + 2 * e) = make_uint2(tile[off], tile[PW + off]);
        }
    };

    uint32_t st = st_first, ti = 0, tj = 0;
    bool act = st < nst && coords(st, ti, tj);
    if (!ts.early) pdl_wait(), pdl_trigger();                           // the previous grid's writes are visible
    if (TMAS) {
        uint4 v[G];
        if (act) load(v, ti, tj);
        if (ts.early) pdl_wait(), pdl_trigger();        // before the first global store
        while (st < nst) {
            const uint32_t si = st / stc, sj = st - si * stc;
            const bool cact = act;
            if (cact) store_tile(v);                     // T1
            __syncwarp();
            st += gridDim.x;
            act = st < nst && coords(st, ti, tj);
            if (act) load(v, ti, tj);                    // T3
            if (threadIdx.x == 0) tma_wait_read();       // the previous TMA store has read staging
            __syncthreads();
            if (cact) drain_staging();                   // T2 into the dense staging tile
            fence_proxy_async();
            __syncthreads();
            if (threadIdx.x == 0)                        // T2: one bulk tensor store per super-tile
                tma_store_2d(&tmap, staging, (int32_t)(si * SR * 32), (int32_t)(sj * SC * 32));
        }
        if (threadIdx.x == 0) tma_wait_all();
    } else if (DEPTH == 1) {
        uint4 v[G];
        if (act) load(v, ti, tj);
        if (ts.early) pdl_wait(), pdl_trigger();        // before the first global store
        while (st < nst) {
            const uint32_t cti = ti, ctj = tj;
            const bool cact = act;
            if (cact) store_tile(v);                     // T1
            __syncwarp();
            st += st_step;
            act = st < nst && coords(st, ti, tj);
            if (act) load(v, ti, tj);                    // T3: next tile in flight
            if (CL > 1) cluster_sync_relaxed();          // drains of the cluster super-tile together
            else if (SR * SC > 1) __syncthreads();       // drains of the super-tile together
            if (cact) drain(cti, ctj);                   // T2
            __syncwarp();
        }
    } else {
        uint4 va[G], vb[G];
        uint32_t ti2 = 0, tj2 = 0;
        if (act) load(va, ti, tj);
        bool act2 = st + gridDim.x < nst && coords(st + gridDim.x, ti2, tj2);
        if (act2) load(vb, ti2, tj2);
        if (ts.early) pdl_wait(), pdl_trigger();        // before the first global store
        while (st < nst) {
            uint32_t cti = ti, ctj = tj;
            bool cact = act;
            if (cact) store_tile(va);
            __syncwarp();
            act = st + 2 * gridDim.x < nst && coords(st + 2 * gridDim.x, ti, tj);
            if (act) load(va, ti, tj);
            if (SR * SC > 1) __syncthreads();
            if (cact) drain(cti, ctj);
            __syncwarp();
            st += gridDim.x;
            if (st >= nst) break;
            cti = ti2; ctj = tj2; cact = act2;
            if (cact) store_tile(vb);
            __syncwarp();
            act2 = st + 2 * gridDim.x < nst && coords(st + 2 * gridDim.x, ti2, tj2);
            if (act2) load(vb, ti2, tj2);
            if (SR * SC > 1) __syncthreads();
            if (cact) drain(cti, ctj);
            __syncwarp();
            st += gridDim.x;
        }
    }
}

// ------------------------------------------------------------------ launchers
// T0 at launch time: RAP's P (and P^-1) / RAS's r for index 0 of `seed`, on the host (the
// rap_rng.cuh functions compiled for the host: the same code as every kernel's draws)
TileShifts tile_shifts(int layout, uint64_t seed) {
    TileShifts t;
    uint32_t a[32];
    memset(&t, 0, sizeof(t));
    const uint32_t w = layout == RAP_LAYOUT_RAP16 ? 16u : 32u;
    if (layout == RAP_LAYOUT_RAP || layout == RAP_LAYOUT_RAP64 || layout == RAP_LAYOUT_RAP16) {
        perm_serial(seed, 0, w, a);
        for (uint32_t i = 0; i < w; ++i) {
            t.sh[i / 4] |= a[i] << (8 * (i % 4));
            t.inv[a[i] / 4] |= i << (8 * (a[i] % 4));
        }
    } else if (layout == RAP_LAYOUT_RAS) {
        ras_serial(seed, 0, w, a);
        for (uint32_t i = 0; i < w; ++i) t.sh[i / 4] |= a[i] << (8 * (i % 4));
    }
    return t;
}

TransposeTuning default_tuning(uint32_t elem_bytes) {
    TransposeTuning t;
    t.sr = elem_bytes == 4 ? kDefaultSR32 : kDefaultSR64;
    t.sc = elem_bytes == 4 ? kDefaultSC32 : kDefaultSC64;
    t.minb = elem_bytes == 4 ? kDefaultMinB32 : kDefaultMinB64;
    t.depth = elem_bytes == 4 ? kDefaultDepth32 : kDefaultDepth64;
    t.ctas_per_sm = elem_bytes == 4 ? kDefaultCtas32 : kDefaultCtas64;
    t.vst = elem_bytes == 4 ? kDefaultVst32 : kDefaultVst64;
    t.cl = elem_bytes == 4 ? kDefaultCL32 : kDefaultCL64;
    return t;
}

// cuTensorMapEncodeTiled through the runtime's driver entry point (no libcuda link dependency)
typedef CUresult (*EncodeTiledFn)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                                  const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static EncodeTiledFn encode_tiled() {
    static EncodeTiledFn fn = [] {
        void *p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) != cudaSuccess ||
            q != cudaDriverEntryPointSuccess)
            p = nullptr;
        return reinterpret_cast<EncodeTiledFn>(p);
    }();
    return fn;
}

// 2-D tensor map of the output (cols rows x rows columns, pitch ld_dst): x = output column (= input
// row), y = output row (= input column); box = one super-tile's output block
static bool make_out_map(CUtensorMap *m, void *dst, int64_t rows, int64_t cols, int64_t ld_dst, int EW,
                         int box_x, int box_y) {
    EncodeTiledFn fn = encode_tiled();
    if (!fn || (uintptr_t)dst % 16 || (ld_dst * EW * 4) % 16) return false;
    const cuuint64_t dims[2] = {(cuuint64_t)rows, (cuuint64_t)cols};
    const cuuint64_t strides[1] = {(cuuint64_t)ld_dst * EW * 4};
    const cuuint32_t box[2] = {(cuuint32_t)box_x, (cuuint32_t)box_y};
    const cuuint32_t estr[2] = {1, 1};
    return fn(m, EW == 1 ? CU_TENSOR_MAP_DATA_TYPE_UINT32 : CU_TENSOR_MAP_DATA_TYPE_UINT64, 2, dst, dims, strides,
              box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
              CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// Cluster launch: as many clusters as can be co-resident (cached per kernel and device), each
// looping over cluster super-tiles.
template <typename K>
static cudaError_t launch_clustered(K kernel, ShapeCache &cache, int cl, int threads, size_t smem, int64_t nst,
                                    cudaStream_t st, const uint32_t *src, uint32_t *dst, int64_t rows, int64_t cols,
                                    int64_t ld_src, int64_t ld_dst, const TileShifts &ts, uint32_t tiles_r,
                                    uint32_t tiles_c, bool vst_ok, const PeerOut &peers, const CUtensorMap &tmap) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    if (dev < 0 || dev >= kMaxDevices) return cudaErrorInvalidDevice;
    int ncl = cache.occ[dev].load(std::memory_order_acquire);   // here: co-resident clusters
    if (ncl == 0) {
        e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        if (cl > 8) {                                            // 16-CTA clusters are non-portable
            e = cudaFuncSetAttribute(kernel, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
            if (e != cudaSuccess) return e;
        }
        int sms = 0;
        e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        if (e != cudaSuccess) return e;
        cudaLaunchConfig_t cfg = {};
        cudaLaunchAttribute attr[1];
        attr[0].id = cudaLaunchAttributeClusterDimension;
        attr[0].val.clusterDim.x = (unsigned)cl;
        attr[0].val.clusterDim.y = 1;
        attr[0].val.clusterDim.z = 1;
        cfg.blockDim = dim3((unsigned)threads);
        cfg.dynamicSmemBytes = smem;
        cfg.attrs = attr;
        cfg.numAttrs = 1;
        cfg.gridDim = dim3((unsigned)(sms * cl));
        e = cudaOccupancyMaxActiveClusters(&ncl, kernel, &cfg);
        if (e != cudaSuccess) return e;
        if (ncl < 1) return cudaErrorInvalidConfiguration;
        cache.occ[dev].store(ncl, std::memory_order_release);
    }
    const int64_t nclusters = nst < ncl ? nst : ncl;
    return launch_ex(kernel, (int)(nclusters * cl), threads, smem, st, cl, src, dst, rows, cols, ld_src, ld_dst, ts,
                     tiles_r, tiles_c, vst_ok, peers, tmap);
}

template <int L, int EW, bool VEC, int DEPTH, int MINB, bool VST, int SR, int SC, bool PEERS = false,
          bool TMAS = false, int CL = 1, bool KP = false>
static cudaError_t launch_one(const void *src, void *dst, int64_t rows, int64_t cols, int64_t ld_src,
                              int64_t ld_dst, uint64_t seed, const TransposeTuning &tu, cudaStream_t st,
                              const PeerOut &peers = PeerOut{}) {
    CUtensorMap tmap;
    memset(&tmap, 0, sizeof(tmap));
    if (TMAS && !make_out_map(&tmap, dst, rows, cols, ld_dst, EW, SR * 32, SC * 32))
        return launch_one<L, EW, VEC, DEPTH, MINB, VST, SR, SC, PEERS, false>(src, dst, rows, cols, ld_src,
                                                                             ld_dst, seed, tu, st, peers);
    const uint32_t tiles_r = (uint32_t)((rows + 31) / 32), tiles_c = (uint32_t)((cols + 31) / 32);
    const int64_t nst = (int64_t)((tiles_r + SR * CL - 1) / (SR * CL)) * ((tiles_c + SC - 1) / SC);
    auto k = transpose_kernel<L, EW, VEC, DEPTH, MINB, VST, SR, SC, PEERS, TMAS, CL, KP>;
    static ShapeCache cache;
    bool vst_ok = ((uintptr_t)dst % 16 == 0) && ((ld_dst * EW * 4) % 16 == 0);
    if (PEERS) {
        vst_ok = ((ld_dst * EW * 4) % 16 == 0) && ((peers.col_off * EW * 4) % 16 == 0);
        for (int h = 0; h < peers.G; ++h) vst_ok = vst_ok && (peers.ptr[h] % 16 == 0);
    }
    const size_t smem = sizeof(uint32_t) * (warp_smem_words<L, EW>() * SR * SC +
                                            (TMAS ? (size_t)SR * 32 * SC * 32 * EW : 0));
    TileShifts ts = tile_shifts(L, seed);
    if (PEERS || KP) pdl_forget(st);
    else ts.early = pdl_early_loads(st, src, rows, cols, ld_src, dst, cols, rows, ld_dst, 4u * EW) ? 1u : 0u;
    if (CL > 1)
        return launch_clustered(k, cache, CL, SR * SC * 32, smem, nst, st, (const uint32_t *)src, (uint32_t *)dst,
                                rows, cols, ld_src, ld_dst, ts, tiles_r, tiles_c, vst_ok, peers, tmap);
    int grid = 0;
    const cudaError_t e = cached_grid(k, cache, SR * SC * 32, smem, nst, tu.ctas_per_sm, &grid);
    if (e != cudaSuccess) return e;
    return launch_ex(k, grid, SR * SC * 32, smem, st, 1, (const uint32_t *)src, (uint32_t *)dst, rows, cols, ld_src,
                     ld_dst, ts, tiles_r, tiles_c, vst_ok, peers, tmap);
}

template <int L, int EW, bool VEC>
static cudaError_t launch_shape(const void *src, void *dst, int64_t rows, int64_t cols, int64_t ld_src,
                                int64_t ld_dst, uint64_t seed, const TransposeTuning &tu, cudaStream_t st) {
#define RAPK_SHAPE(D, M, V, R_, C_)                                                                  \
    if (tu.depth == D && tu.minb == M && tu.vst == V && tu.sr == R_ && tu.sc == C_ && !tu.tma_store && tu.cl == 1) \
        return launch_one<L, EW, VEC, D, M, V, R_, C_>(src, dst, rows, cols, ld_src, ld_dst, seed, tu, st);
#define RAPK_TSHAPE(M, R_, C_)                                                                       \
    if (tu.depth == 1 && tu.minb == M && !tu.vst && tu.sr == R_ && tu.sc == C_ && tu.tma_store && tu.cl == 1) \
        return launch_one<L, EW, VEC, 1, M, false, R_, C_, false, true>(src, dst, rows, cols, ld_src, ld_dst, \
                                                                        seed, tu, st);
#ifdef RAP_TUNING_SWEEP
    RAPK_SHAPE(1, 1, false, 4, 1) RAPK_SHAPE(1, 4, false, 4, 1) RAPK_SHAPE(1, 3, false, 4, 1)
    RAPK_SHAPE(1, 1, false, 8, 1) RAPK_SHAPE(1, 2, false, 8, 1) RAPK_SHAPE(1, 3, false, 8, 1)
    RAPK_SHAPE(1, 1, false, 16, 1) RAPK_SHAPE(1, 2, false, 16, 1) RAPK_SHAPE(2, 1, false, 16, 1)
    RAPK_SHAPE(1, 1, false, 8, 2) RAPK_SHAPE(1, 1, false, 12, 1) RAPK_SHAPE(1, 1, true, 16, 1)
    RAPK_SHAPE(2, 2, false, 8, 1) RAPK_SHAPE(1, 1, false, 6, 1) RAPK_SHAPE(1, 2, false, 6, 1)
    RAPK_SHAPE(2, 1, false, 8, 2) RAPK_SHAPE(2, 1, false, 4, 2) RAPK_SHAPE(1, 1, false, 4, 4)
    RAPK_SHAPE(2, 1, false, 4, 4) RAPK_SHAPE(1, 1, true, 8, 2) RAPK_SHAPE(2, 1, false, 12, 1)
    RAPK_TSHAPE(1, 8, 2) RAPK_TSHAPE(1, 8, 1) RAPK_TSHAPE(1, 4, 2) RAPK_TSHAPE(1, 4, 1) RAPK_TSHAPE(1, 4, 4)
    RAPK_TSHAPE(2, 4, 2) RAPK_TSHAPE(2, 8, 1)
#endif
#undef RAPK_SHAPE
#undef RAPK_TSHAPE
    (void)tu;
    // a handful of tiles (cfg1's single 32 x 32 tile): one warp per CTA, one CTA per tile -- no
    // cluster, no idle warps of a super-tile computing P, the cheapest launch
    if (((rows + 31) / 32) * ((cols + 31) / 32) <= kSmallTiles)
        return launch_one<L, EW, VEC, 1, 1, false, 1, 1>(src, dst, rows, cols, ld_src, ld_dst, seed, tu, st);
    // column-pair slots (RAP32_PAIR): 32-bit elements as virtual 8-byte elements (a[i][2k], a[i][2k+1])
    // through the one-double-per-slot kernel (transpose64.cu)
    if constexpr (EW == 1 && VEC) {
        if (RAP32_PAIR && tu.cl == kDefaultCL32 && cols % 2 == 0 && ld_src % 2 == 0)
            return launch_transpose_pair32(src, dst, rows, cols, ld_src, ld_dst, L, seed, st);
    }
    // row-pair planes (KP): 32-bit elements as virtual 8-byte elements, the 64-bit kernel's shape
    if constexpr (EW == 1 && VEC) {
        if (RAP32_KP && tu.cl == kDefaultCL32 && rows % 2 == 0 && ld_dst % 2 == 0 && (uintptr_t)dst % 8 == 0)
            return launch_one<L, 2, true, 1, RAP32_KP_MINB, false, RAP32_KP_SR, 1, false, false, RAP32_KP_CL, true>(
                src, dst, rows / 2, cols, ld_src, ld_dst / 2, seed, tu, st);
    }
    if (EW == 1 && tu.cl == kDefaultCL32)
        return launch_one<L, EW, VEC, kDefaultDepth32, kDefaultMinB32, kDefaultVst32, kDefaultSR32, kDefaultSC32,
                          false, false, kDefaultCL32>(src, dst, rows, cols, ld_src, ld_dst, seed, tu, st);
    if (EW == 1)      // the round-1 shape without cluster (8 x 2 warps), kept selectable for A/B runs
        return launch_one<L, EW, VEC, 1, 1, false, 8, 2>(src, dst, rows, cols, ld_src, ld_dst, seed, tu, st);
    return launch_one<L, EW, VEC, kDefaultDepth64, kDefaultMinB64, kDefaultVst64, kDefaultSR64, kDefaultSC64,
                      false, false, kDefaultCL64>(src, dst, rows, cols, ld_src, ld_dst, seed, tu, st);
}

template <bool VEC>
static cudaError_t dispatch(const void *src, void *dst, int64_t rows, int64_t cols, int64_t ld_src,
                            int64_t ld_dst, uint32_t eb, int layout, uint64_t seed,
                            const TransposeTuning &tu, cudaStream_t st) {
    // 64-bit elements: RAW..RAP on two 32-bit planes (this kernel, EW = 2); RAP64 keeps one
    // element per 8-byte slot (transpose64.cu, which also serves RAW..RAS with tu.slots64)
    if (eb == 8 && layout == RAP_LAYOUT_RAP64)
        return launch_transpose64(src, dst, rows, cols, ld_src, ld_dst, RAP_LAYOUT_RAP, seed, st);
    if (eb == 8 && tu.slots64)
        return launch_transpose64(src, dst, rows, cols, ld_src, ld_dst, layout, seed, st);
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

template <bool VEC>
static cudaError_t dispatch_peers(const void *src, int64_t rows, int64_t cols, int64_t ld_src, int64_t ld_dst,
                                  uint32_t eb, int layout, uint64_t seed, const PeerOut &pe, cudaStream_t st) {
    const TransposeTuning tu = default_tuning(eb);
#define RAPK_PEER(LAY)                                                                              \
    case LAY:                                                                                       \
        return eb == 4                                                                              \
            ? launch_one<LAY, 1, VEC, kDefaultDepth32, 1, kDefaultVst32, kPeerSR32,                  \
                         kPeerSC32, true>(src, nullptr, rows, cols, ld_src, ld_dst, seed, tu, st, pe)   \
            : launch_one<LAY, 2, VEC, kDefaultDepth64, kDefaultMinB64, kDefaultVst64, kDefaultSR64,  \
                         kDefaultSC64, true>(src, nullptr, rows, cols, ld_src, ld_dst, seed, tu, st, pe);
    switch (layout) {
        RAPK_PEER(RAP_LAYOUT_RAW)
        RAPK_PEER(RAP_LAYOUT_PAD)
        RAPK_PEER(RAP_LAYOUT_XOR)
        RAPK_PEER(RAP_LAYOUT_RAS)
        RAPK_PEER(RAP_LAYOUT_RAP)
    }
#undef RAPK_PEER
    return cudaErrorInvalidValue;
}

cudaError_t launch_transpose_peers(const void *src, int64_t M, int64_t N, int64_t ld_src, const PeerOut &pe,
                                   int64_t ld_dst, uint32_t elem_bytes, int layout, uint64_t seed, cudaStream_t st) {
    const bool vec = ((uintptr_t)src % 16 == 0) && ((ld_src * elem_bytes) % 16 == 0);
    return vec ? dispatch_peers<true>(src, M, N, ld_src, ld_dst, elem_bytes, layout, seed, pe, st)
               : dispatch_peers<false>(src, M, N, ld_src, ld_dst, elem_bytes, layout, seed, pe, st);
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
    if (layout == RAP_LAYOUT_RAP16)
        return elem_bytes == 8 ? launch_transpose_rap16(src, dst, rows, cols, ld_src, ld_dst, seed, st)
                               : cudaErrorInvalidValue;
    return launch_transpose_tuned(src, dst, rows, cols, ld_src, ld_dst, elem_bytes, layout, seed,
                                  default_tuning(elem_bytes), st);
}

}  // namespace rapk
