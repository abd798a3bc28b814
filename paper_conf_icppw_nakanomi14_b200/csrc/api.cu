// api.cu -- the extern "C" boundary of librap.so (include/rap.h): argument validation on the
// host, then one enqueue of the corresponding kernel launcher.  No computation of the method
// happens here; there is no CPU fallback.
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/rap.h"
#include "rap_internal.h"
#include "rap_rng.cuh"

namespace {

rap_status_t from_cuda(cudaError_t e) { return e == cudaSuccess ? RAP_OK : RAP_ERR_CUDA; }

bool is_pow2(uint32_t w) { return w && !(w & (w - 1)); }

// product of two non-negative int64 without overflow -> false on overflow
bool mul_ok(int64_t a, int64_t b, int64_t *out) {
    if (a < 0 || b < 0) return false;
    if (a != 0 && b > INT64_MAX / a) return false;
    *out = a * b;
    return true;
}

// byte extent [first, last) touched by a row-major matrix with leading dimension ld
bool extent(uintptr_t base, int64_t rows, int64_t cols, int64_t ld, uint32_t eb, uintptr_t *lo,
            uintptr_t *hi) {
    int64_t span;
    if (!mul_ok(rows - 1, ld, &span)) return false;
    if (span > INT64_MAX - cols) return false;
    span += cols;
    int64_t bytes;
    if (!mul_ok(span, (int64_t)eb, &bytes)) return false;
    *lo = base;
    *hi = base + (uintptr_t)bytes;
    return *hi >= *lo;
}

}  // namespace

extern "C" {

int rap_abi_version(void) { return RAP_ABI_VERSION; }

const char *rap_status_str(rap_status_t s) {
    switch (s) {
    case RAP_OK: return "RAP_OK";
    case RAP_ERR_INVALID_ARG: return "RAP_ERR_INVALID_ARG: argument out of range";
    case RAP_ERR_UNSUPPORTED: return "RAP_ERR_UNSUPPORTED: request not implemented";
    case RAP_ERR_ALIAS: return "RAP_ERR_ALIAS: src and dst overlap (transpose is out-of-place)";
    case RAP_ERR_CUDA: return "RAP_ERR_CUDA: CUDA runtime or launch failure";
    }
    return "RAP_ERR_UNKNOWN";
}

rap_status_t rap_perm_gen(uint64_t seed, uint64_t index, uint32_t w, uint32_t *perm_out) {
    if (w < 2 || w > RAP_MAX_W_SWEEP || !perm_out) return RAP_ERR_INVALID_ARG;
    rapk::perm_serial(seed, index, w, perm_out);
    return RAP_OK;
}

rap_status_t rap_perm_gen_batch(uint64_t seed, uint64_t first_index, uint64_t count, uint32_t w,
                                uint8_t *d_perm_out, void *stream) {
    if (w < 2 || w > RAP_MAX_W) return RAP_ERR_INVALID_ARG;
    if (count == 0) return RAP_OK;
    if (!d_perm_out || count > (UINT64_MAX / w)) return RAP_ERR_INVALID_ARG;
    return from_cuda(rapk::launch_perm_gen(seed, first_index, count, w, d_perm_out,
                                           (cudaStream_t)stream));
}

rap_status_t rap_transpose(const void *src, void *dst, int64_t rows, int64_t cols, int64_t ld_src,
                           int64_t ld_dst, uint32_t elem_bytes, rap_layout_t layout, uint64_t seed,
                           void *stream) {
    if (elem_bytes != 4 && elem_bytes != 8) return RAP_ERR_INVALID_ARG;
    if ((int)layout < RAP_LAYOUT_RAW || (int)layout > RAP_LAYOUT_RAP64) return RAP_ERR_INVALID_ARG;
    if ((layout == RAP_LAYOUT_RAP16 || layout == RAP_LAYOUT_RAP64) && elem_bytes != 8) return RAP_ERR_UNSUPPORTED;
    if (rows < 0 || cols < 0) return RAP_ERR_INVALID_ARG;
    if (rows == 0 || cols == 0) return RAP_OK;
    if (!src || !dst) return RAP_ERR_INVALID_ARG;
    if (ld_src < cols || ld_dst < rows) return RAP_ERR_INVALID_ARG;
    if ((uintptr_t)src % elem_bytes || (uintptr_t)dst % elem_bytes) return RAP_ERR_INVALID_ARG;
    uintptr_t s_lo, s_hi, d_lo, d_hi;
    if (!extent((uintptr_t)src, rows, cols, ld_src, elem_bytes, &s_lo, &s_hi) ||
        !extent((uintptr_t)dst, cols, rows, ld_dst, elem_bytes, &d_lo, &d_hi))
        return RAP_ERR_INVALID_ARG;
    if (s_lo < d_hi && d_lo < s_hi) return RAP_ERR_ALIAS;
    // 32 x 32 tiles are indexed with 32-bit counters: up to 2^31 tiles (2^41 elements)
    if (((rows + 31) / 32) * ((cols + 31) / 32) >= (int64_t(1) << 31)) return RAP_ERR_UNSUPPORTED;
    return from_cuda(rapk::launch_transpose(src, dst, rows, cols, ld_src, ld_dst, elem_bytes,
                                            (int)layout, seed, (cudaStream_t)stream));
}

rap_status_t rap_transpose_host(const void *h_src, void *h_dst, int64_t rows, int64_t cols, int64_t ld_src,
                                int64_t ld_dst, uint32_t elem_bytes, rap_layout_t layout, uint64_t seed,
                                void *d_workspace, size_t workspace_bytes, void *stream) {
    if (elem_bytes != 4 && elem_bytes != 8) return RAP_ERR_INVALID_ARG;
    if ((int)layout < RAP_LAYOUT_RAW || (int)layout > RAP_LAYOUT_RAP64) return RAP_ERR_INVALID_ARG;
    if ((layout == RAP_LAYOUT_RAP16 || layout == RAP_LAYOUT_RAP64) && elem_bytes != 8) return RAP_ERR_UNSUPPORTED;
    if (rows < 0 || cols < 0) return RAP_ERR_INVALID_ARG;
    if (rows == 0 || cols == 0) return RAP_OK;
    if (!h_src || !h_dst || !d_workspace) return RAP_ERR_INVALID_ARG;
    if (ld_src < cols || ld_dst < rows) return RAP_ERR_INVALID_ARG;
    uintptr_t s_lo, s_hi, d_lo, d_hi;
    if (!extent((uintptr_t)h_src, rows, cols, ld_src, elem_bytes, &s_lo, &s_hi) ||
        !extent((uintptr_t)h_dst, cols, rows, ld_dst, elem_bytes, &d_lo, &d_hi))
        return RAP_ERR_INVALID_ARG;
    if (s_lo < d_hi && d_lo < s_hi) return RAP_ERR_ALIAS;
    if (rapk::host_band_rows(rows, cols, elem_bytes, workspace_bytes) == 0) return RAP_ERR_INVALID_ARG;
    return from_cuda(rapk::transpose_host(h_src, h_dst, rows, cols, ld_src, ld_dst, elem_bytes, (int)layout, seed,
                                          d_workspace, workspace_bytes, (cudaStream_t)stream));
}

rap_status_t rap_transpose_to_peers(const void *src, int64_t M, int64_t N, int64_t ld_src,
                                    void *const *peer_dst, uint32_t G, uint32_t rank, int64_t ld_dst,
                                    uint32_t elem_bytes, rap_layout_t layout, uint64_t seed, void *stream) {
    if (elem_bytes != 4 && elem_bytes != 8) return RAP_ERR_INVALID_ARG;
    if ((int)layout < RAP_LAYOUT_RAW || (int)layout > RAP_LAYOUT_RAP64) return RAP_ERR_INVALID_ARG;
    if (layout == RAP_LAYOUT_RAP16 || layout == RAP_LAYOUT_RAP64) return RAP_ERR_UNSUPPORTED;
    if (G < 1 || G > (uint32_t)rapk::kMaxPeers || rank >= G || !peer_dst) return RAP_ERR_INVALID_ARG;
    if (M <= 0 || M % 32 != 0) return RAP_ERR_INVALID_ARG;
    int64_t gm;
    if (!mul_ok((int64_t)G, M, &gm) || N != gm) return RAP_ERR_INVALID_ARG;
    if (!src || ld_src < N || ld_dst < N) return RAP_ERR_INVALID_ARG;
    if ((uintptr_t)src % elem_bytes) return RAP_ERR_INVALID_ARG;
    rapk::PeerOut pe;
    pe.G = (int)G;
    pe.M = M;
    pe.col_off = (int64_t)rank * M;
    uintptr_t s_lo, s_hi;
    if (!extent((uintptr_t)src, M, N, ld_src, elem_bytes, &s_lo, &s_hi)) return RAP_ERR_INVALID_ARG;
    for (uint32_t h = 0; h < G; ++h) {
        if (!peer_dst[h] || (uintptr_t)peer_dst[h] % elem_bytes) return RAP_ERR_INVALID_ARG;
        uintptr_t d_lo, d_hi;
        if (!extent((uintptr_t)peer_dst[h], M, N, ld_dst, elem_bytes, &d_lo, &d_hi)) return RAP_ERR_INVALID_ARG;
        if (s_lo < d_hi && d_lo < s_hi) return RAP_ERR_ALIAS;
        pe.ptr[h] = (uint64_t)(uintptr_t)peer_dst[h];
    }
    if ((M / 32) * ((N + 31) / 32) >= (int64_t(1) << 31)) return RAP_ERR_UNSUPPORTED;
    return from_cuda(rapk::launch_transpose_peers(src, M, N, ld_src, pe, ld_dst, elem_bytes, (int)layout,
                                                  seed, (cudaStream_t)stream));
}

rap_status_t rap_congestion(uint32_t w, uint64_t n_warps, const uint32_t *d_rows,
                            const uint32_t *d_cols, rap_scheme_t scheme, const uint32_t *d_shift,
                            uint32_t *d_congestion_out, void *stream) {
    if (w < 2 || w > RAP_MAX_W) return RAP_ERR_INVALID_ARG;
    if ((int)scheme < RAP_SCHEME_RAW || (int)scheme > RAP_SCHEME_XOR) return RAP_ERR_INVALID_ARG;
    if (scheme == RAP_SCHEME_XOR && !is_pow2(w)) return RAP_ERR_INVALID_ARG;
    if (n_warps == 0) return RAP_OK;
    if (!d_rows || !d_cols || !d_congestion_out) return RAP_ERR_INVALID_ARG;
    if ((scheme == RAP_SCHEME_RAS || scheme == RAP_SCHEME_RAP) && !d_shift) return RAP_ERR_INVALID_ARG;
    if (n_warps > UINT64_MAX / w) return RAP_ERR_INVALID_ARG;
    const uint32_t *shift = (scheme == RAP_SCHEME_RAS || scheme == RAP_SCHEME_RAP) ? d_shift : nullptr;
    return from_cuda(rapk::launch_congestion(w, n_warps, d_rows, d_cols, (int)scheme, shift,
                                             d_congestion_out, (cudaStream_t)stream));
}

rap_status_t rap_congestion_sweep_algo(uint32_t w, uint32_t pattern_mask, uint32_t scheme_mask,
                                       uint64_t seed, uint64_t first_trial, uint64_t n_trials,
                                       uint64_t *d_hist, uint32_t algo, void *stream) {
    if (w < 2 || w > RAP_MAX_W_SWEEP) return RAP_ERR_INVALID_ARG;
    if (algo > RAP_SWEEP_MATCH) return RAP_ERR_INVALID_ARG;
    if (w > RAP_MAX_W && algo != RAP_SWEEP_DEFAULT) return RAP_ERR_UNSUPPORTED;
    if (pattern_mask == 0 || pattern_mask > 31u || scheme_mask == 0 || scheme_mask > 31u)
        return RAP_ERR_INVALID_ARG;
    if (((scheme_mask >> RAP_SCHEME_XOR) & 1u) && !is_pow2(w)) return RAP_ERR_INVALID_ARG;
    if (n_trials == 0) return RAP_OK;
    if (!d_hist) return RAP_ERR_INVALID_ARG;
    auto launch = w > RAP_MAX_W ? rapk::launch_sweep_wide
                : algo == RAP_SWEEP_MATCH ? rapk::launch_sweep_match : rapk::launch_sweep;
    return from_cuda(launch(w, pattern_mask, scheme_mask, seed, first_trial, n_trials, d_hist,
                            (cudaStream_t)stream));
}

rap_status_t rap_congestion_sweep(uint32_t w, uint32_t pattern_mask, uint32_t scheme_mask,
                                  uint64_t seed, uint64_t first_trial, uint64_t n_trials,
                                  uint64_t *d_hist, void *stream) {
    return rap_congestion_sweep_algo(w, pattern_mask, scheme_mask, seed, first_trial, n_trials,
                                     d_hist, RAP_SWEEP_DEFAULT, stream);
}

rap_status_t rap_congestion_sweep4(uint32_t w, uint32_t pattern_mask, uint32_t scheme_mask, uint64_t seed,
                                   uint64_t first_trial, uint64_t n_trials, uint64_t *d_hist, void *stream) {
    if (w < 4 || w > RAP_MAX_W) return RAP_ERR_INVALID_ARG;
    if (pattern_mask == 0 || pattern_mask > 63u || scheme_mask == 0 || scheme_mask > 31u)
        return RAP_ERR_INVALID_ARG;
    if (n_trials == 0) return RAP_OK;
    if (!d_hist) return RAP_ERR_INVALID_ARG;
    return from_cuda(rapk::launch_sweep4(w, pattern_mask, scheme_mask, seed, first_trial, n_trials, d_hist,
                                         (cudaStream_t)stream));
}

rap_status_t rap_congestion_trace(uint32_t w, uint64_t n_warps, const uint32_t *d_cells,
                                  uint32_t scheme_mask, uint64_t seed, uint64_t first_trial,
                                  uint64_t n_trials, uint64_t *d_hist, void *stream) {
    if (w < 2 || w > RAP_MAX_W) return RAP_ERR_INVALID_ARG;
    if (scheme_mask == 0 || scheme_mask > 31u) return RAP_ERR_INVALID_ARG;
    if (((scheme_mask >> RAP_SCHEME_XOR) & 1u) && !is_pow2(w)) return RAP_ERR_INVALID_ARG;
    if (n_warps == 0 || n_trials == 0) return RAP_OK;
    if (!d_cells || !d_hist) return RAP_ERR_INVALID_ARG;
    if (n_warps > UINT64_MAX / w) return RAP_ERR_INVALID_ARG;
    return from_cuda(rapk::launch_trace(w, n_warps, d_cells, scheme_mask, seed, first_trial,
                                        n_trials, d_hist, (cudaStream_t)stream));
}

rap_status_t rap_unpack_blocks(const void *d_recv, void *d_out, int64_t G, int64_t M, int64_t ld_out,
                               uint32_t elem_bytes, void *stream) {
    if (elem_bytes != 4 && elem_bytes != 8) return RAP_ERR_INVALID_ARG;
    if (G < 0 || M < 0) return RAP_ERR_INVALID_ARG;
    if (G == 0 || M == 0) return RAP_OK;
    int64_t width;
    if (!mul_ok(G, M, &width) || ld_out < width) return RAP_ERR_INVALID_ARG;
    if (!d_recv || !d_out) return RAP_ERR_INVALID_ARG;
    if ((uintptr_t)d_recv % elem_bytes || (uintptr_t)d_out % elem_bytes) return RAP_ERR_INVALID_ARG;
    uintptr_t r_lo, r_hi, o_lo, o_hi;
    int64_t rrows;
    if (!mul_ok(G, M, &rrows)) return RAP_ERR_INVALID_ARG;
    if (!extent((uintptr_t)d_recv, rrows, M, M, elem_bytes, &r_lo, &r_hi) ||
        !extent((uintptr_t)d_out, M, width, ld_out, elem_bytes, &o_lo, &o_hi))
        return RAP_ERR_INVALID_ARG;
    if (r_lo < o_hi && o_lo < r_hi) return RAP_ERR_ALIAS;
    return from_cuda(rapk::launch_unpack_blocks(d_recv, d_out, G, M, ld_out, elem_bytes, (cudaStream_t)stream));
}

rap_status_t rap_smem_transpose_bench(uint32_t algorithm, rap_scheme_t scheme, uint32_t elem_bytes,
                                      uint64_t seed, uint32_t n_blocks, uint32_t reps, uint32_t *d_out,
                                      uint64_t *d_cycles, void *stream) {
    if (algorithm > RAP_DRDW) return RAP_ERR_INVALID_ARG;
    if (scheme != RAP_SCHEME_RAW && scheme != RAP_SCHEME_RAS && scheme != RAP_SCHEME_RAP) return RAP_ERR_INVALID_ARG;
    if (elem_bytes != 4 && elem_bytes != 8) return RAP_ERR_INVALID_ARG;
    if (n_blocks == 0) return RAP_OK;
    if (n_blocks > (1u << 24) || !d_out || !d_cycles) return RAP_ERR_INVALID_ARG;
    return from_cuda(rapk::launch_smem_bench(algorithm, (int)scheme, elem_bytes, seed, n_blocks, reps, d_out,
                                             d_cycles, (cudaStream_t)stream));
}

rap_status_t rap_smem_gather_bench(const uint16_t *d_src_index, rap_layout_t layout, uint64_t seed,
                                   uint32_t n_blocks, uint32_t reps, uint32_t *d_out, uint64_t *d_cycles,
                                   void *stream) {
    if ((int)layout < RAP_LAYOUT_RAW || (int)layout > RAP_LAYOUT_RAP) return RAP_ERR_INVALID_ARG;
    if (n_blocks == 0) return RAP_OK;
    if (n_blocks > (1u << 24) || !d_src_index || !d_out || !d_cycles) return RAP_ERR_INVALID_ARG;
    return from_cuda(rapk::launch_smem_gather(d_src_index, (int)layout, seed, n_blocks, reps, d_out, d_cycles,
                                              (cudaStream_t)stream));
}

}  // extern "C"
