// pdl_registry.cu -- which transpose ran last in each stream (host side of early loads under
// programmatic dependent launch; rap_internal.h pdl_early_loads).
#include <cuda_runtime.h>
#include <stdint.h>

#include <mutex>

#include "rap_internal.h"

namespace rapk {

namespace {

struct Entry {
    int dev = -1;
    cudaStream_t st = nullptr;
    uintptr_t lo = 0, hi = 0;   // the last transpose's destination byte range in this stream
    bool valid = false;
};
constexpr int kEntries = 64;
std::mutex g_mu;
Entry g_tab[kEntries];
int g_next = 0;

// byte extent of a row-major matrix (the caller validated the sizes)
void extent(const void *p, int64_t rows, int64_t cols, int64_t ld, uint32_t eb, uintptr_t *lo, uintptr_t *hi) {
    *lo = (uintptr_t)p;
    *hi = *lo + (uintptr_t)(((rows - 1) * ld + cols) * (int64_t)eb);
}

Entry *find(int dev, cudaStream_t st) {
    for (auto &e : g_tab)
        if (e.dev == dev && e.st == st) return &e;
    return nullptr;
}

}  // namespace

// RAP_PDL_EARLY (default 0): whether early loads are used at all.  The registry knows the last
// transpose launched in a stream, not the last kernel: a third-party kernel launched in between
// with programmatic dependent launch of its own (CUTLASS / GEMM libraries trigger early) could
// still be writing this launch's source -- so early loads stay off unless a build opts in.
#ifndef RAP_PDL_EARLY
#define RAP_PDL_EARLY 0
#endif

bool pdl_early_loads(cudaStream_t st, const void *src, int64_t rows, int64_t cols, int64_t ld_src, const void *dst,
                     int64_t drows, int64_t dcols, int64_t ld_dst, uint32_t eb) {
    if (!RAP_PDL || !RAP_PDL_EARLY) return false;
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return false;
    uintptr_t s_lo, s_hi, d_lo, d_hi;
    extent(src, rows, cols, ld_src, eb, &s_lo, &s_hi);
    extent(dst, drows, dcols, ld_dst, eb, &d_lo, &d_hi);
    std::lock_guard<std::mutex> lock(g_mu);
    Entry *e = find(dev, st);
    // the legacy / per-thread default streams synchronise with other streams: stay conservative
    const bool known = e && e->valid && st != nullptr && st != cudaStreamLegacy && st != cudaStreamPerThread;
    const bool early = known && (s_hi <= e->lo || e->hi <= s_lo);
    if (!e) {
        e = &g_tab[g_next];
        g_next = (g_next + 1) % kEntries;   // (an evicted stream just loses its early loads)
        e->dev = dev;
        e->st = st;
    }
    e->lo = d_lo;
    e->hi = d_hi;
    e->valid = true;
    return early;
}

void pdl_forget(cudaStream_t st) {
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return;
    std::lock_guard<std::mutex> lock(g_mu);
    if (Entry *e = find(dev, st)) e->valid = false;
}

}  // namespace rapk
