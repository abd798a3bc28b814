/*
 * rap.h -- C ABI of librap.so, the B200 (sm_100a) hot path of the Random Address
 * Permute-Shift (RAP) technique of Nakano, Matsumae and Ito (ICPPW 2014).
 *
 * Citations "P:L<a>-<b>" are line numbers in the paper text plus the section,
 * figure or table.  The problem statement these calls follow (§II):
 *   - the Discrete Memory Machine (DMM) has w memory banks; address a is in bank a mod w;
 *   - a warp of w threads issues w requests at once; identical addresses are merged;
 *   - the congestion of the access is the maximum number of distinct requests destined
 *     for one bank.
 * RAP stores element a[i][j] of a w x w matrix at a[i][(j + P[i]) mod w] for a permutation
 * P drawn uniformly from all w! permutations (§IV, Fig.6); RAS is the same with
 * independent shifts r[i]; RAW is the plain row-major layout.
 *
 * Conventions (all entry points):
 *   - Ownership: the caller owns every buffer.  Pointers named d_* (and src/dst of
 *     rap_transpose) are DEVICE pointers on the current CUDA device.  The library keeps no
 *     memory allocation and no shared mutable state; calls are thread-safe.  (Cached per
 *     kernel: the launch shape; per calling thread and device: rap_transpose_host's three
 *     streams and their events, created on first use and destroyed at thread exit; in builds
 *     with RAP_PDL_EARLY only, a mutex-guarded table of the last transpose per stream.)
 *   - Asynchrony: device work is enqueued on `stream` (a cudaStream_t passed as void*;
 *     NULL = the legacy default stream) and returns immediately; results are valid once
 *     the stream is synchronised.
 *   - Errors: argument errors are detected on the host BEFORE anything is enqueued and
 *     returned as RAP_ERR_INVALID_ARG / RAP_ERR_UNSUPPORTED / RAP_ERR_ALIAS; a failed
 *     launch returns RAP_ERR_CUDA.  No exception crosses the ABI.  There is no CPU
 *     fallback: every computation runs in the library's CUDA kernels.
 *   - Random numbers (paper: "selected uniformly at random"; the contract is
 *     this library's, reading vi): Philox4x32-10 with key = (seed_lo, seed_hi);
 *     word t of domain d for index n is Philox(ctr = (n_lo, n_hi, t>>2, d), key)[t & 3].
 *     Domain 0 feeds the permutation (Durstenfeld: for k = w-1..1, j = floor(word(0,w-1-k)
 *     * (k+1) / 2^32), swap a[k], a[j]); domain 1 the RAS shifts r[i] = floor(word(1,i) *
 *     w / 2^32); domain 2 the random-access cells cell_t = floor(word(2,t) * w*w / 2^32).
 */
#ifndef RAP_H_
#define RAP_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define RAP_ABI_VERSION 2
#define RAP_MAX_W 32          /* warp-wide evaluators: one CUDA warp = one DMM warp          */
#define RAP_MAX_W_SWEEP 256   /* rap_congestion_sweep: 32 < w <= 256 spans one CUDA warp over  */
                              /* w/32 request slices (sweep_wide.cu)                          */

typedef enum {
    RAP_OK = 0,
    RAP_ERR_INVALID_ARG = 1,  /* a size, pointer, enum or mask is out of range          */
    RAP_ERR_UNSUPPORTED = 2,  /* valid request this build does not implement             */
    RAP_ERR_ALIAS = 3,        /* src and dst of an out-of-place transpose overlap        */
    RAP_ERR_CUDA = 4          /* a CUDA runtime call or kernel launch failed             */
} rap_status_t;

/* Shared-memory tile layouts of rap_transpose (a 32 x 32 tile, row i of the input tile). */
typedef enum {
    RAP_LAYOUT_RAW = 0,  /* a[i][j] at [i][j]                   (RAW CRSW)   */
    RAP_LAYOUT_PAD = 1,  /* a[i][j] at [i][j] of a [32][33] array   (+1 padding baseline) */
    RAP_LAYOUT_XOR = 2,  /* a[i][j] at [i][j xor i]                 (XOR-swizzle baseline)*/
    RAP_LAYOUT_RAS = 3,  /* a[i][j] at [i][(j + r[i]) mod 32]          */
    RAP_LAYOUT_RAP = 4,  /* a[i][j] at [i][(j + P[i]) mod 32]        */
    RAP_LAYOUT_RAP16 = 5,/* 64-bit elements only (else RAP_ERR_UNSUPPORTED): a tile of     */
                         /* doubles with one element per PAIR of 4-byte banks, i.e. 16   */
                         /* "double banks"; a[i][j] at [i][16*(j div 16) + ((j + Q[i mod */
                         /* 16]) mod 16)], Q = perm(seed, 0, 16).  The paper's RAP with  */
                         /* w = 16 applied to each half row: every half-warp of a 64-bit */
                         /* row or column access hits 16 distinct bank pairs (P:L860,    */
                         /* L1005-1023, DESIGN reading xiv)            */
    RAP_LAYOUT_RAP64 = 6 /* 64-bit elements only: the paper's map a[i][(j + P[i]) mod 32] */
                         /* with ONE double per 8-byte tile slot, as the paper's arrays of */
                         /* doubles (where a bank held one double).  B200 banks */
                         /* are 4 bytes, so a 64-bit access is served per half-warp (16     */
                         /* doubles); the kernel assigns rows to lanes so that every half-  */
                         /* warp of the row write and of the column read hits 16 distinct  */
                         /* bank pairs (DESIGN reading xv)                                 */
} rap_layout_t;
/* With elem_bytes == 8, RAW..RAP split each 64-bit element into two 32-bit planes (low words,
 * high words) with identical addressing, so every shared-memory access is a 32-lane 4-byte access
 * under the w = 32 map of the layout (DESIGN reading viii). */

/* Address maps of the DMM congestion evaluator (physical address of logical cell (i,j)). */
typedef enum {
    RAP_SCHEME_RAW = 0,  /* i*w + j                                                      */
    RAP_SCHEME_RAS = 1,  /* i*w + (j + r[i]) mod w                                       */
    RAP_SCHEME_RAP = 2,  /* i*w + (j + P[i]) mod w                                       */
    RAP_SCHEME_PAD = 3,  /* i*(w+1) + j                                                  */
    RAP_SCHEME_XOR = 4   /* i*w + (j xor i); w must be a power of two                    */
} rap_scheme_t;

/* Warp access patterns of the sweep; lane t = 0..w-1 (§III). */
typedef enum {
    RAP_PAT_CONTIGUOUS = 0,  /* (0, t)                                                    */
    RAP_PAT_STRIDE = 1,      /* (t, 0)                                                    */
    RAP_PAT_DIAGONAL = 2,    /* (t, t)       Fig.4 warp W(0): a[(0+t) mod w][t]           */
    RAP_PAT_RANDOM = 3,      /* w cells i.i.d. uniform with replacement (domain 2)        */
    RAP_PAT_MALICIOUS = 4    /* scheme-aware worst case: RAW,RAS -> (t,0); RAP,XOR ->     */
                             /* (t,t); PAD -> (t,(w-t) mod w)       (reading iii)*/
} rap_pattern_t;

/* §VII: schemes and warp patterns of a w x w x w x w array (NEXT-3). */
typedef enum {
    RAP_SCHEME4_RAW = 0,  /* f = 0                                                        */
    RAP_SCHEME4_RAS = 1,  /* f = r[i][j][k], w^3 independent shifts (domain 1, index (i*w+j)*w+k) */
    RAP_SCHEME4_1P = 2,   /* f = P[k]                                  (One permutation)   */
    RAP_SCHEME4_R1P = 3,  /* f = P[i] + P[j] + P[k] mod w              (Repeated one perm.)*/
    RAP_SCHEME4_3P = 4    /* f = P[i] + Q[j] + R[k] mod w; Q, R from domains 3, 4 (3 perms) */
} rap_scheme4_t;

typedef enum {
    RAP_PAT4_CONTIGUOUS = 0,  /* a[0][0][0][t]                                            */
    RAP_PAT4_STRIDE1 = 1,     /* a[0][0][t][0]                                            */
    RAP_PAT4_STRIDE2 = 2,     /* a[0][t][0][0]                                            */
    RAP_PAT4_STRIDE3 = 3,     /* a[t][0][0][0]                                            */
    RAP_PAT4_RANDOM = 4,      /* w cells of w^4 i.i.d. with replacement (domain 2)        */
    RAP_PAT4_MALICIOUS = 5    /* RAW, RAS: stride1; 1P: stride2; R1P, 3P: floor(w/6) groups of */
                              /* the 6 permutations of (3g, 3g+1, 3g+2) at l = 0;  */
                              /* remaining lanes repeat lane 0's request (merged)          */
} rap_pattern4_t;

int rap_abi_version(void);
const char *rap_status_str(rap_status_t s);

/* T0 -- one permutation P = perm(seed, index, w) of {0..w-1}, on the HOST (P:L316-320, L959-962
 * §IV: "P is selected uniformly at random from all w! permutations"; the counter contract above
 * fixes which one).  perm_out: host uint32_t[w], caller-owned; 2 <= w <= 256 (Table II's widths).
 * Deterministic and synchronous; no GPU involved.  This is how every transpose launch obtains
 * its P (index 0): computed once per call on the host and passed to the kernel by value
 * (the paper: the random numbers are "computed beforehand"). */
rap_status_t rap_perm_gen(uint64_t seed, uint64_t index, uint32_t w, uint32_t *perm_out);

/* T0, batched on the device -- P_n = perm(seed, n, w) for n = first_index .. first_index+count-1.
 * d_perm_out: device uint8_t[count][w]; row k holds P_{first_index+k}.  2 <= w <= 32; one warp
 * per permutation (warp Fisher-Yates, one shuffle per swap).  count == 0 is a no-op. */
rap_status_t rap_perm_gen_batch(uint64_t seed, uint64_t first_index, uint64_t count, uint32_t w,
                                uint8_t *d_perm_out, void *stream);

/* T1-T3 -- out-of-place transpose staged through 32 x 32 shared-memory tiles in `layout`
 * (§III; RAP layout P:L1005-1023 §IV, RAP CRSW listing P:L1515-1546 §VI):
 *     dst[c * ld_dst + r] = src[r * ld_src + c]   for 0 <= r < rows, 0 <= c < cols.
 * src, dst: device pointers, row-major with leading dimensions ld_src >= cols and
 * ld_dst >= rows (elements).  elem_bytes in {4, 8}: a raw bit copy (float32/float64 NaN
 * payloads, -0, subnormals are preserved).  The tile layout changes only where an element
 * sits in shared memory, never the result.  RAP uses P = perm(seed, 0, 32), RAS uses
 * r = shifts(seed, 0, 32), both computed on the host at launch (rap_perm_gen); seed is ignored
 * by RAW/PAD/XOR.  rows == 0 or cols == 0 is a
 * no-op.  Overlapping src/dst -> RAP_ERR_ALIAS.  16-byte aligned src with ld_src a
 * multiple of 16/elem_bytes takes 128-bit loads; anything else takes 32/64-bit loads
 * (still on the GPU).  RAP_LAYOUT_RAP16 and RAP_LAYOUT_RAP64 (elem_bytes 8 only) are the
 * other 64-bit encodings of T2b. */
rap_status_t rap_transpose(const void *src, void *dst, int64_t rows, int64_t cols,
                           int64_t ld_src, int64_t ld_dst, uint32_t elem_bytes,
                           rap_layout_t layout, uint64_t seed, void *stream);

/* T1-T3 from and to HOST memory (the end-to-end call): dst = src^T as rap_transpose, but src
 * and dst are HOST pointers (pinned memory lets the copies overlap).  The matrix moves in row
 * bands of a multiple of 32 rows: upload of band b+1, transpose of band b and 2-D download of
 * band b-1 run concurrently on three internal streams (PCIe in both directions at once); band
 * heights ramp up at the start and down at the end so the pipeline fills and drains quickly.
 * d_workspace: caller-owned DEVICE buffer of workspace_bytes; it holds 4 band buffers, so it must
 * fit at least 4 * 32 * cols * elem_bytes bytes (larger = fewer, longer bands).  The call is
 * SYNCHRONOUS: work queued on `stream` before the call completes first, and dst is valid on
 * return.  Errors as rap_transpose (+ RAP_ERR_INVALID_ARG for a too-small workspace). */
rap_status_t rap_transpose_host(const void *h_src, void *h_dst, int64_t rows, int64_t cols, int64_t ld_src,
                                int64_t ld_dst, uint32_t elem_bytes, rap_layout_t layout, uint64_t seed,
                                void *d_workspace, size_t workspace_bytes, void *stream);

/* T4, fused (NEXT-2) -- the row-block-sharded N x N transpose without the all-to-all: rank
 * `rank` of G holds rows rank*M .. rank*M+M-1 of A (src: M x N, ld_src >= N, N = G*M, M a
 * multiple of 32) and writes every 32 x 32 output tile straight into the output shard of the
 * rank that owns it:
 *     peer_dst[h][(c - h*M) * ld_dst + rank*M + r] = src[r * ld_src + c],   h = c / M,
 * so out_h = rows h*M .. h*M+M-1 of A^T.  peer_dst: HOST array of G device pointers valid in
 * this process (peer shards mapped over NVLink -- CUDA IPC / symmetric memory -- or local
 * buffers for a one-GPU emulation); ld_dst >= N; G <= 16.  One HBM read and one NVLink write
 * per element; no send/receive buffers, no unpack.  Enqueue only: the caller must make every
 * rank's kernel complete (a cross-rank barrier) before reading its output shard.
 * layout RAW..RAP (RAP16 / RAP64 -> RAP_ERR_UNSUPPORTED); 64-bit elements are staged as two
 * 32-bit planes. */
rap_status_t rap_transpose_to_peers(const void *src, int64_t M, int64_t N, int64_t ld_src,
                                    void *const *peer_dst, uint32_t G, uint32_t rank, int64_t ld_dst,
                                    uint32_t elem_bytes, rap_layout_t layout, uint64_t seed, void *stream);

/* C3 -- the DMM congestion evaluator itself (§II), batched: warp k issues the w
 * requests to logical cells (d_rows[k*w + t], d_cols[k*w + t]) of a w x w matrix laid out
 * by `scheme` with per-warp shift vector d_shift[k*w .. k*w+w-1] (P for RAP, r for RAS;
 * may be NULL for RAW/PAD/XOR).  d_congestion_out[k] = max over banks of the number of
 * distinct addresses destined for the bank (1..w).  Cells and shifts must be < w; a warp
 * with any out-of-range cell or shift gets congestion 0 (an error marker, never a valid
 * congestion).  n_warps == 0 is a no-op. */
rap_status_t rap_congestion(uint32_t w, uint64_t n_warps, const uint32_t *d_rows,
                            const uint32_t *d_cols, rap_scheme_t scheme, const uint32_t *d_shift,
                            uint32_t *d_congestion_out, void *stream);

/* C1-C4 -- Monte-Carlo sweep (Tab.II P:L1567-1577 §V): for every trial n in
 * [first_trial, first_trial + n_trials) draw P_n, r_n and the random cells from the counter
 * contract, evaluate each selected (pattern, scheme) and count the congestion.
 * d_hist: device uint64_t[npat][nsch][w+1] where npat = popcount(pattern_mask) and
 * nsch = popcount(scheme_mask), patterns/schemes in enum order; ACCUMULATED (+=), so the
 * caller zeroes it once and may split a run into any chunks (bit-identical sums).
 * Masks are bit sets of rap_pattern_t / rap_scheme_t (1..31).  XOR needs w = 2^k.
 * 2 <= w <= RAP_MAX_W_SWEEP (256, Table II's widths): w <= 32 maps a DMM warp onto a CUDA warp;
 * 32 < w <= 256 (NEXT-3; RAP_SWEEP_DEFAULT only) gives a CUDA warp a batch of 32 trials: each
 * lane runs one trial's Durstenfeld chain, then lane L plays DMM threads L + 32i of one trial at
 * a time (merged requests by __match_any_sync + a w*w-bit bitmap, bank counts by shared atomics). */
rap_status_t rap_congestion_sweep(uint32_t w, uint32_t pattern_mask, uint32_t scheme_mask,
                                  uint64_t seed, uint64_t first_trial, uint64_t n_trials,
                                  uint64_t *d_hist, void *stream);

/* NEXT-3 -- §VII Monte-Carlo sweep over a w^4 array (Table IV): trial n draws
 * P, Q, R (domains 0, 3, 4), the random cells (domain 2) and the RAS shifts it needs (domain 1)
 * and counts the congestion of each selected (rap_pattern4_t, rap_scheme4_t).  4 <= w <= 32;
 * pattern_mask 1..63, scheme_mask 1..31; d_hist: device uint64_t[npat][nsch][w+1], ACCUMULATED. */
rap_status_t rap_congestion_sweep4(uint32_t w, uint32_t pattern_mask, uint32_t scheme_mask, uint64_t seed,
                                   uint64_t first_trial, uint64_t n_trials, uint64_t *d_hist, void *stream);

/* Kernel designs of the sweep (identical histograms):
 *   RAP_SWEEP_DEFAULT  lane-mode bit-sliced Fisher-Yates (one trial per lane, no shuffles)
 *                      + ballot bank histogram in warp mode;
 *   RAP_SWEEP_MATCH    one warp per trial, shuffle Fisher-Yates + __match_any_sync histogram
 *                      (kept as the measured ablation). */
typedef enum { RAP_SWEEP_DEFAULT = 0, RAP_SWEEP_MATCH = 1 } rap_sweep_algo_t;

/* rap_congestion_sweep with an explicit kernel design; algo outside rap_sweep_algo_t ->
 * RAP_ERR_INVALID_ARG.  rap_congestion_sweep(...) == rap_congestion_sweep_algo(..., 0, ...). */
rap_status_t rap_congestion_sweep_algo(uint32_t w, uint32_t pattern_mask, uint32_t scheme_mask,
                                       uint64_t seed, uint64_t first_trial, uint64_t n_trials,
                                       uint64_t *d_hist, uint32_t algo, void *stream);

/* C3 over user traces: d_cells: device uint32_t[n_warps][w], cell = row*w + col < w*w.
 * Every trace warp is evaluated under every trial's P_n / r_n, n in [first_trial,
 * first_trial + n_trials).  d_hist: device uint64_t[nsch][w+1], ACCUMULATED (+=);
 * each scheme row gains n_warps * n_trials counts.  Bin 0 counts trace warps holding a
 * cell >= w*w (invalid input; valid congestions are 1..w). */
rap_status_t rap_congestion_trace(uint32_t w, uint64_t n_warps, const uint32_t *d_cells,
                                  uint32_t scheme_mask, uint64_t seed, uint64_t first_trial,
                                  uint64_t n_trials, uint64_t *d_hist, void *stream);

/* T4 -- block unpack after the all-to-all of the row-block-sharded transpose (BASELINE cfg5;
 * not in the paper, which has one w x w matrix).  Rank g of G holds rows gM..(g+1)M of the
 * N x N matrix A (N = G*M); rap_transpose of that M x N shard gives N x M whose row block s is
 * the M x M block destined for rank s; after the exchange the receive buffer holds, for every
 * source s, recv[s] = (A[sM:(s+1)M, gM:(g+1)M])^T (M x M, contiguous, source order).  This call
 * places it:  d_out[x * ld_out + s*M + a] = d_recv[(s*M + x) * M + a]  (0 <= s < G, x, a < M),
 * i.e. rows gM..(g+1)M of A^T.  Device pointers; ld_out >= G*M; raw bit copy of elem_bytes in
 * {4, 8}; overlapping buffers -> RAP_ERR_ALIAS; G == 0 or M == 0 is a no-op. */
rap_status_t rap_unpack_blocks(const void *d_recv, void *d_out, int64_t G, int64_t M, int64_t ld_out,
                               uint32_t elem_bytes, void *stream);

/* NEXT-1 -- the paper's experiment (Table III, §VI) on this GPU: a 32 x 32 matrix
 * transposed `reps` times between two shared-memory arrays by one CTA of 1024 threads, with
 * algorithm CRSW / SRCW / DRDW (§III) under layout RAW / RAS / RAP (both arrays laid
 * out, reading v).  CTA k uses P = perm(seed, k, 32) or r = shifts(seed, k, 32).
 * d_out: device uint32_t[n_blocks][1024], logical element (i, j) of the final array (initial
 * a[i][j] = 32 i + j, so the result is the identity for even reps and the transpose for odd);
 * d_cycles: device uint64_t[n_blocks], SM clock cycles of the timed loop (reps transposes, each
 * followed by __syncthreads).  elem_bytes 4 or 8 (the paper used 8-byte doubles in 8-byte bank
 * mode; B200 banks are 4 bytes).  ncu's shared wavefronts per request over many CTAs is the
 * hardware's expected congestion of each access. */
typedef enum { RAP_CRSW = 0, RAP_SRCW = 1, RAP_DRDW = 2 } rap_smem_algorithm_t;
rap_status_t rap_smem_transpose_bench(uint32_t algorithm, rap_scheme_t scheme, uint32_t elem_bytes,
                                      uint64_t seed, uint32_t n_blocks, uint32_t reps, uint32_t *d_out,
                                      uint64_t *d_cycles, void *stream);

/* NEXT-4 -- a data-dependent shared-memory access under a given layout (the paper's motivation:
 * addresses not known beforehand).  One CTA of 1024 threads applies the
 * tile permutation `reps` times inside shared memory: thread o writes element o (row o/32,
 * contiguous) from source element d_src_index[o] of the previous array (a gather), for
 * o = 0..1023.  d_src_index: device uint16_t[1024], values < 1024 (need not be a permutation;
 * the host cannot validate device data, so the kernel uses each index mod 1024).
 * Layouts: RAW, PAD [32][33], XOR [i][j^i], RAS, RAP; CTA k uses P/r of (seed, k).
 * d_out: device uint32_t[n_blocks][1024] final array (initial value of element o is o), i.e.
 * out[o] = src^reps(o); d_cycles: device uint64_t[n_blocks] SM cycles of the timed loop. */
rap_status_t rap_smem_gather_bench(const uint16_t *d_src_index, rap_layout_t layout, uint64_t seed,
                                   uint32_t n_blocks, uint32_t reps, uint32_t *d_out, uint64_t *d_cycles,
                                   void *stream);

#ifdef __cplusplus
}
#endif

#endif /* RAP_H_ */
