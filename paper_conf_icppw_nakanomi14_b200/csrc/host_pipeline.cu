// host_pipeline.cu -- rap_transpose_host: the transpose of a HOST matrix into a HOST matrix,
// pipelined over row bands so that PCIe runs both directions at once.
//
//   band b (rows b*RB .. b*RB+RB-1 of src):  H2D (stream in)  ->  rap_transpose kernel
//   (stream compute)  ->  2-D D2H of the cols x RB result into columns b*RB.. of dst (stream out)
//
// Two device buffers per direction (double buffering) live in the caller's workspace; events
// order the three streams, so band b+1 is uploading while band b is transposed and band b-1 is
// downloading.  Band heights ramp (RB/4, RB/2, then RB) at the start and back down
// at the end, so the pipeline fills (first upload) and drains (last download) on small bands
// while the middle runs in full-size bands.  The call is synchronous: it returns once dst holds the result.  Host buffers
// should be pinned (page-locked) for the copies to overlap; pageable memory still works.
#include <cuda_runtime.h>
#include <stdint.h>

#include <memory>
#include <vector>

#include "rap_internal.h"

namespace rapk {

namespace {

struct Streams {
    cudaStream_t s[3] = {nullptr, nullptr, nullptr};
    cudaEvent_t ev[3][2] = {};
    cudaEvent_t start = nullptr;
    cudaError_t err = cudaSuccess;
    Streams() {
        err = cudaEventCreateWithFlags(&start, cudaEventDisableTiming);
        for (auto &x : s)
            if (err == cudaSuccess) err = cudaStreamCreateWithFlags(&x, cudaStreamNonBlocking);
        for (auto &row : ev)
            for (auto &e : row)
                if (err == cudaSuccess) err = cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
    }
    ~Streams() {
        if (start) cudaEventDestroy(start);
        for (auto &row : ev)
            for (auto &e : row)
                if (e) cudaEventDestroy(e);
        for (auto &x : s)
            if (x) cudaStreamDestroy(x);
    }
};

}  // namespace

size_t host_band_rows(int64_t rows, int64_t cols, uint32_t eb, size_t work_bytes) {
    // 4 buffers of band_rows x cols elements; bands a multiple of 32 rows (whole tiles)
    const size_t per_row = (size_t)cols * eb * 4;
    if (per_row == 0) return 0;
    size_t rb = work_bytes / per_row;
    rb = rb / 32 * 32;
    const size_t cap = (size_t)((rows + 31) / 32 * 32);
    return rb < cap ? rb : cap;
}

// Band heights for `rows` rows with full bands of rb rows: a doubling ramp from rb/4 (at least
// 32 rows) up to rb at the head, full bands in the middle, the mirrored ramp at the tail.
#ifndef RAP_HOST_RAMP_DIV
#define RAP_HOST_RAMP_DIV 4    // smallest ramp band = rb / RAP_HOST_RAMP_DIV (0: no ramp); narrower bands
                               // make the strided download slow (256 B of each 32 KiB row: 32 GB/s)
#endif
static std::vector<int64_t> band_plan(int64_t rows, int64_t rb, uint32_t eb) {
    std::vector<int64_t> head;
    int64_t ramp = 0;
    int64_t s0 = RAP_HOST_RAMP_DIV ? rb / RAP_HOST_RAMP_DIV / 32 * 32 : rb;
    // a band of s rows downloads as `cols` segments of s * eb bytes; ramp bands below 1 KiB
    // segments cost more than the shorter fill saves (cfg4 at a 64 MiB workspace: 91 GB/s without
    // the 256 / 512-byte ramp bands, 85 with them; profiles/r02_e2e_bands.txt)
    const int64_t min_rows = (1024 / eb + 31) / 32 * 32;
    if (s0 < min_rows) s0 = min_rows;
    for (int64_t s = s0 < 32 ? 32 : s0; s < rb; s *= 2) {
        head.push_back(s);
        ramp += s;
    }
    std::vector<int64_t> plan;
    if (rows < 2 * ramp + rb) {                       // too small to ramp: equal bands
        for (int64_t r = 0; r < rows; r += rb) plan.push_back(rows - r < rb ? rows - r : rb);
        return plan;
    }
    plan = head;
    int64_t mid = rows - 2 * ramp;
    const int64_t rem = mid % rb;
    if (rem) plan.push_back(rem);                     // the ragged full-size band first
    for (mid -= rem; mid > 0; mid -= rb) plan.push_back(rb);
    for (auto it = head.rbegin(); it != head.rend(); ++it) plan.push_back(*it);
    return plan;
}

cudaError_t transpose_host(const void *h_src, void *h_dst, int64_t rows, int64_t cols, int64_t ld_src,
                           int64_t ld_dst, uint32_t eb, int layout, uint64_t seed, void *d_work,
                           size_t work_bytes, cudaStream_t user) {
    const size_t rb = host_band_rows(rows, cols, eb, work_bytes);
    if (rb == 0) return cudaErrorInvalidValue;
    // the three streams and their events are created once per (thread, device) and reused: creating
    // them per call cost ~0.3 ms, 4 % of a cfg3 host-to-host transpose
    int dev = 0;
    cudaError_t de = cudaGetDevice(&dev);
    if (de != cudaSuccess) return de;
    if (dev < 0 || dev >= kMaxDevices) return cudaErrorInvalidDevice;
    thread_local std::unique_ptr<Streams> cache[kMaxDevices];
    if (!cache[dev] || cache[dev]->err != cudaSuccess) cache[dev].reset(new Streams());
    Streams &st = *cache[dev];
    if (st.err != cudaSuccess) return st.err;
    cudaStream_t s_in = st.s[0], s_cmp = st.s[1], s_out = st.s[2];
    // order after whatever the caller queued on its stream
    cudaEvent_t start = st.start;
    cudaError_t e = cudaEventRecord(start, user);
    if (e != cudaSuccess) return e;
    for (cudaStream_t x : {s_in, s_cmp, s_out}) cudaStreamWaitEvent(x, start, 0);
    const size_t band_bytes = rb * (size_t)cols * eb;
    uint8_t *din[2] = {(uint8_t *)d_work, (uint8_t *)d_work + band_bytes};
    uint8_t *dout[2] = {(uint8_t *)d_work + 2 * band_bytes, (uint8_t *)d_work + 3 * band_bytes};
    const std::vector<int64_t> plan = band_plan(rows, (int64_t)rb, eb);
    const int64_t nb = (int64_t)plan.size();
    int64_t r0 = 0;
    for (int64_t b = 0; b < nb && e == cudaSuccess; r0 += plan[b], ++b) {
        const int k = (int)(b & 1);
        const int64_t nr = plan[b];
        // H2D: buffer k is free once the transpose of band b-2 has consumed it
        if (b >= 2) cudaStreamWaitEvent(s_in, st.ev[1][k], 0);
        e = cudaMemcpy2DAsync(din[k], (size_t)cols * eb, (const uint8_t *)h_src + (size_t)r0 * ld_src * eb,
                              (size_t)ld_src * eb, (size_t)cols * eb, (size_t)nr, cudaMemcpyHostToDevice, s_in);
        if (e != cudaSuccess) break;
        cudaEventRecord(st.ev[0][k], s_in);
        // transpose: needs the upload, and out buffer k drained by the D2H of band b-2
        cudaStreamWaitEvent(s_cmp, st.ev[0][k], 0);
        if (b >= 2) cudaStreamWaitEvent(s_cmp, st.ev[2][k], 0);
        e = launch_transpose(din[k], dout[k], nr, cols, cols, nr, eb, layout, seed, s_cmp);
        if (e != cudaSuccess) break;
        cudaEventRecord(st.ev[1][k], s_cmp);
        // D2H: cols rows of nr elements into columns r0 .. r0+nr-1 of dst
        cudaStreamWaitEvent(s_out, st.ev[1][k], 0);
        e = cudaMemcpy2DAsync((uint8_t *)h_dst + (size_t)r0 * eb, (size_t)ld_dst * eb, dout[k], (size_t)nr * eb,
                              (size_t)nr * eb, (size_t)cols, cudaMemcpyDeviceToHost, s_out);
        if (e != cudaSuccess) break;
        cudaEventRecord(st.ev[2][k], s_out);
    }
    cudaError_t e2 = cudaStreamSynchronize(s_out);
    cudaStreamSynchronize(s_in);
    cudaStreamSynchronize(s_cmp);
    return e != cudaSuccess ? e : e2;
}

}  // namespace rapk
