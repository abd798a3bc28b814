// rap_internal.h -- launcher declarations shared by the kernel translation units and the
// C-ABI layer (api.cu).  Not part of the public ABI (include/rap.h).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>

#include "../../include/rap.h"

namespace rapk {

constexpr int kMaxDevices = 64;
constexpr int kMaxPeers = 16;

// T0 at launch time: the shift vector of the tile layout, computed once per call on the host
// (perm_serial / ras_serial of rap_rng.cuh, index 0) and passed to the kernel by value, so no
// warp spends its prologue on Philox + Fisher-Yates.  RAP: sh = P, inv = P^-1; RAP-16: sh = Q
// (w = 16) and inv = Q^-1; RAS: sh = r.  Unused for RAW / PAD / XOR.
struct TileShifts {
    uint32_t sh[8];    // byte i of the 32-byte vector = sh[i / 4] >> (8 * (i % 4))
    uint32_t inv[8];
    uint32_t early = 0;  // 1: the grid may load its source before the previous grid completes
                         // (pdl_early_loads); it still waits before its first global store
};

// byte i (< 32) of a packed TileShifts vector: uniform constant-bank words + a per-lane select
// (a dynamic index into a kernel parameter would copy the struct to local memory)
__device__ __forceinline__ uint32_t shift_byte(const uint32_t (&w)[8], uint32_t i) {
    // the words are first moved into registers through opaque movs: otherwise the compiler
    // recognises the select chain as an indexed parameter access and lowers THAT to a
    // predicated walk over the whole struct, once per use
    uint32_t r[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) asm("mov.b32 %0, %1;" : "=r"(r[k]) : "r"(w[k]));
    const uint32_t q = i >> 2;
    const uint32_t a = (q & 1u) ? r[1] : r[0], b = (q & 1u) ? r[3] : r[2];
    const uint32_t c = (q & 1u) ? r[5] : r[4], d = (q & 1u) ? r[7] : r[6];
    const uint32_t ab = (q & 2u) ? b : a, cd = (q & 2u) ? d : c;
    const uint32_t x = (q & 4u) ? cd : ab;
    return (x >> (8u * (i & 3u))) & 0xffu;
}
TileShifts tile_shifts(int layout, uint64_t seed);

// Launch shape cached per kernel instantiation and device: the dynamic-smem attribute and the
// occupancy query run once.  `occ` (0 = unknown) is published with release after `sms`, and
// read with acquire, so a reader that sees occ != 0 also sees sms.
struct ShapeCache {
    std::atomic<int> occ[kMaxDevices];
    std::atomic<int> sms[kMaxDevices];
};

// Fused-exchange output (NEXT-2): the output shard base of each of the G ranks, as pointers
// valid in this process (mapped peer memory), M = rows per rank, col_off = rank * M.
struct PeerOut {
    uint64_t ptr[kMaxPeers] = {};
    int64_t M = 1;
    int64_t col_off = 0;
    int G = 0;
};

// Launch-shape knobs of the transpose (defaults chosen by tools/tune_transpose.cu on B200).
struct TransposeTuning {
    int sr = 4, sc = 1;   // super-tile of sr x sc tiles per CTA, one warp per tile, lockstep
    int minb = 2;         // __launch_bounds__ min blocks per SM (register budget)
    int depth = 1;        // tiles of global loads in flight per warp (register double-buffer)
    int ctas_per_sm = 0;  // persistent grid = #SMs x this (0: as many as fit)
    bool vst = false;     // 128-bit output stores (shuffle-transposed) instead of 32/64-bit rows
    bool tma_store = false;  // drain into a dense staging tile, one TMA bulk tensor store per super-tile
    int cl = 1;           // thread-block cluster of cl CTAs stacked along the input rows, drains in lockstep
    bool slots64 = false;  // 64-bit elements on 8-byte tile slots (transpose64.cu) for every layout (A/B)
};
// fp32: 4 x 2 warps per CTA, clusters of 8 CTAs (a 32 x 2-tile cluster super-tile: each output
// row receives 4 KiB per drain; +1.5 % over clusters of 4 with PDL off, profiles/r02_ab32s3.txt);
// fp64: 12 x 1 warps, no cluster (profiles/r01_tune_transpose*.txt, r01_probe_transpose.txt)
// (RAP32_SR / RAP32_SC / RAP32_CL / RAP32_MINB override the fp32 shape in tuning builds)
#ifndef RAP32_SR
#define RAP32_SR 4
#endif
#ifndef RAP32_SC
#define RAP32_SC 2
#endif
#ifndef RAP32_CL
#define RAP32_CL 8
#endif
#ifndef RAP32_MINB
#define RAP32_MINB 2
#endif
// (RAP64P_SR / RAP64P_CL / RAP64P_MINB: the two-plane fp64 shape in tuning builds)
#ifndef RAP64P_SR
#define RAP64P_SR 12
#endif
#ifndef RAP64P_CL
#define RAP64P_CL 1
#endif
#ifndef RAP64P_MINB
#define RAP64P_MINB 1
#endif
constexpr int kDefaultSR32 = RAP32_SR, kDefaultSC32 = RAP32_SC, kDefaultSR64 = RAP64P_SR, kDefaultSC64 = 1;
constexpr int kDefaultCL32 = RAP32_CL, kDefaultCL64 = RAP64P_CL;
// fused sharded transpose (peer stores): 8 x 2 warps, no cluster
constexpr int kPeerSR32 = 8, kPeerSC32 = 2;
// up to this many 32 x 32 tiles: one single-warp CTA per tile
constexpr int64_t kSmallTiles = 8;
// measured on B200 (tools/tune_transpose.cu, profiles/r01_tune_transpose.txt)
constexpr int kDefaultMinB32 = RAP32_MINB, kDefaultMinB64 = RAP64P_MINB;   // fp32: 2 CTAs of 8 warps per SM (128 registers)
constexpr int kDefaultDepth32 = 1, kDefaultDepth64 = 1;
constexpr int kDefaultCtas32 = 0, kDefaultCtas64 = 0;
constexpr bool kDefaultVst32 = false, kDefaultVst64 = false;
TransposeTuning default_tuning(uint32_t elem_bytes);

cudaError_t launch_transpose_tuned(const void *src, void *dst, int64_t rows, int64_t cols, int64_t ld_src,
                                   int64_t ld_dst, uint32_t elem_bytes, int layout, uint64_t seed,
                                   const TransposeTuning &tu, cudaStream_t st);

cudaError_t launch_transpose(const void *src, void *dst, int64_t rows, int64_t cols, int64_t ld_src,
                             int64_t ld_dst, uint32_t elem_bytes, int layout, uint64_t seed,
                             cudaStream_t st);

cudaError_t launch_transpose_rap16(const void *src, void *dst, int64_t rows, int64_t cols, int64_t ld_src,
                                   int64_t ld_dst, uint64_t seed, cudaStream_t st);

// 64-bit elements, one element per 8 bytes of the tile (transpose64.cu): layouts RAW..RAP
cudaError_t launch_transpose64(const void *src, void *dst, int64_t rows, int64_t cols, int64_t ld_src,
                               int64_t ld_dst, int layout, uint64_t seed, cudaStream_t st);

// 32-bit elements as column-pair 8-byte slots (transpose64.cu; tuning path RAP32_PAIR of transpose.cu)
cudaError_t launch_transpose_pair32(const void *src, void *dst, int64_t rows, int64_t cols, int64_t ld_src,
                                    int64_t ld_dst, int layout, uint64_t seed, cudaStream_t st);

cudaError_t launch_transpose_peers(const void *src, int64_t M, int64_t N, int64_t ld_src, const PeerOut &pe,
                                   int64_t ld_dst, uint32_t elem_bytes, int layout, uint64_t seed, cudaStream_t st);

cudaError_t launch_perm_gen(uint64_t seed, uint64_t first, uint64_t count, uint32_t w, uint8_t *out,
                            cudaStream_t st);

// Programmatic dependent launch (RAP_PDL, default OFF): the transposes can be launched with
// cudaLaunchAttributeProgrammaticStreamSerialization; they then wait (griddepcontrol.wait) for the
// previous grid in the stream -- its completion and memory flush -- before their first global
// access and trigger their own dependents after that wait, so a following launch's CTAs are
// scheduled and run their prologue while this grid drains; the data dependence is kept.  Measured
// over 21 interleaved rounds (profiles/r02_ab_pdl32b.txt, r02_ab_pdl64b.txt): -4 to -5 % on
// back-to-back cfg3 fp32 launches (clustered grids, much wider spread) and +0.4 % on cfg4 fp64
// (noise) -- so it is off; the kernels' wait / trigger instructions are no-ops without it.
#ifndef RAP_PDL
#define RAP_PDL 0
#endif
__device__ __forceinline__ void pdl_wait() {
#if RAP_PDL
    asm volatile("griddepcontrol.wait;" ::: "memory");
#endif
}
__device__ __forceinline__ void pdl_trigger() {
#if RAP_PDL
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
#endif
}

// Early loads under programmatic dependent launch.  A transpose grid waits for its predecessor
// in the stream (griddepcontrol.wait) before its first global STORE always (write-after-read and
// write-after-write on the previous grid's buffers), and before its first LOAD unless the library
// knows the predecessor: when the previous kernel in this stream was one of these transposes and
// its destination does not overlap this launch's source, nothing this grid reads is being written,
// so its first tiles are loaded while the previous grid drains.  (A kernel of anyone else in
// between is not PDL-aware: this grid then starts after it completes, which covers that case.)
// A grid triggers its dependents (launch_dependents) only after its own wait has returned, so when
// a dependent starts, every grid before this one has completed and only this one may still be
// running: comparing against the previous launch's destination is enough.
// pdl_early_loads() answers for a launch and records its destination for the next one;
// pdl_forget() marks a stream's last kernel as unknown (the fused peer-store transpose).
bool pdl_early_loads(cudaStream_t st, const void *src, int64_t rows, int64_t cols, int64_t ld_src, const void *dst,
                     int64_t drows, int64_t dcols, int64_t ld_dst, uint32_t eb);
void pdl_forget(cudaStream_t st);

// cudaLaunchKernelEx with an optional cluster dimension and the PDL attribute
template <typename K, typename... Args>
cudaError_t launch_ex(K kernel, int grid, int block, size_t smem, cudaStream_t st, int cluster, Args... args) {
    cudaLaunchConfig_t cfg = {};
    cudaLaunchAttribute attr[2];
    int na = 0;
    if (cluster > 1) {
        attr[na].id = cudaLaunchAttributeClusterDimension;
        attr[na].val.clusterDim.x = (unsigned)cluster;
        attr[na].val.clusterDim.y = 1;
        attr[na].val.clusterDim.z = 1;
        ++na;
    }
#if RAP_PDL
    attr[na].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[na].val.programmaticStreamSerializationAllowed = 1;
    ++na;
#endif
    cfg.gridDim = dim3((unsigned)grid);
    cfg.blockDim = dim3((unsigned)block);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cfg.attrs = attr;
    cfg.numAttrs = na;
    const cudaError_t e = cudaLaunchKernelEx(&cfg, kernel, args...);
    return e != cudaSuccess ? e : cudaGetLastError();
}

// occupancy-capped persistent grid for `want` work units (ShapeCache above)
template <typename K>
cudaError_t cached_grid(K kernel, ShapeCache &cache, int threads, size_t smem, int64_t want, int ctas_per_sm,
                        int *grid_out) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    if (dev < 0 || dev >= kMaxDevices) return cudaErrorInvalidDevice;
    int occ = cache.occ[dev].load(std::memory_order_acquire);
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
        cache.occ[dev].store(occ, std::memory_order_release);
    }
    if (ctas_per_sm > 0 && ctas_per_sm < occ) occ = ctas_per_sm;
    const int64_t cap = (int64_t)sms * occ;
    *grid_out = (int)(want < cap ? want : cap);
    return cudaSuccess;
}

cudaError_t launch_congestion(uint32_t w, uint64_t n_warps, const uint32_t *rows, const uint32_t *cols,
                              int scheme, const uint32_t *shift, uint32_t *out, cudaStream_t st);

cudaError_t launch_sweep(uint32_t w, uint32_t pattern_mask, uint32_t scheme_mask, uint64_t seed,
                         uint64_t first, uint64_t n_trials, uint64_t *hist, cudaStream_t st);

cudaError_t launch_sweep_match(uint32_t w, uint32_t pattern_mask, uint32_t scheme_mask, uint64_t seed,
                               uint64_t first, uint64_t n_trials, uint64_t *hist, cudaStream_t st);

cudaError_t launch_sweep_wide(uint32_t w, uint32_t pattern_mask, uint32_t scheme_mask, uint64_t seed,
                              uint64_t first, uint64_t n_trials, uint64_t *hist, cudaStream_t st);

cudaError_t launch_sweep4(uint32_t w, uint32_t pattern_mask, uint32_t scheme_mask, uint64_t seed,
                          uint64_t first, uint64_t n_trials, uint64_t *hist, cudaStream_t st);

cudaError_t launch_trace(uint32_t w, uint64_t n_warps, const uint32_t *cells, uint32_t scheme_mask,
                         uint64_t seed, uint64_t first, uint64_t n_trials, uint64_t *hist,
                         cudaStream_t st);

cudaError_t launch_unpack_blocks(const void *recv, void *out, int64_t G, int64_t M, int64_t ld_out,
                                 uint32_t elem_bytes, cudaStream_t st);

cudaError_t launch_smem_bench(uint32_t alg, int scheme, uint32_t elem_bytes, uint64_t seed, uint32_t n_blocks,
                              uint32_t reps, uint32_t *out, uint64_t *cycles, cudaStream_t st);

cudaError_t launch_smem_gather(const uint16_t *src_index, int layout, uint64_t seed, uint32_t n_blocks,
                               uint32_t reps, uint32_t *out, uint64_t *cycles, cudaStream_t st);

size_t host_band_rows(int64_t rows, int64_t cols, uint32_t eb, size_t work_bytes);
cudaError_t transpose_host(const void *h_src, void *h_dst, int64_t rows, int64_t cols, int64_t ld_src,
                           int64_t ld_dst, uint32_t eb, int layout, uint64_t seed, void *d_work,
                           size_t work_bytes, cudaStream_t user);

}  // namespace rapk
