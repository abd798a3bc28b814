// tune_transpose.cu -- dev harness: times the transpose kernels of librap under launch-shape
// variants (register budget via __launch_bounds__ min blocks, tile traversal group) on the
// BASELINE cfg3 / cfg4 matrices, next to a device-to-device memcpy of the same bytes.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 \
//          -Ipaper_conf_icppw_nakanomi14_b200/csrc -o tools/tune_transpose tools/tune_transpose.cu
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <algorithm>
#include <string>
#define RAP_TUNING_SWEEP 1
#include "transpose.cu"

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e), __LINE__); exit(1);} } while (0)

__global__ void fill(uint32_t *p, size_t n, uint32_t salt) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
        uint32_t x = (uint32_t)i * 2654435761u ^ salt ^ (uint32_t)(i >> 32);
        x ^= x >> 16; x *= 0x7feb352du; x ^= x >> 15; x *= 0x846ca68bu; x ^= x >> 16;
        p[i] = x;
    }
}

__global__ void check_t(const uint32_t *a, const uint32_t *b, int64_t n, int words, unsigned long long *bad) {
    // b (n x n elements of `words` u32) must be the transpose of a
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n * n; i += (int64_t)gridDim.x * blockDim.x) {
        int64_t r = i / n, c = i % n;
        for (int w = 0; w < words; ++w)
            if (a[(r * n + c) * words + w] != b[(c * n + r) * words + w]) { atomicAdd(bad, 1ull); return; }
    }
}

// ---- probes: the tile skeleton without the transpose (same loads, row-wise stores)
template <int DEPTH>
__global__ void __launch_bounds__(128) tilecopy_kernel(const uint32_t *__restrict__ src, uint32_t *__restrict__ dst,
                                                       int64_t n, uint32_t tiles_c, uint32_t ntiles) {
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    const uint32_t q = lane & 7u, c_in = lane >> 3;
    uint32_t t = blockIdx.x * 4 + warp;
    const uint32_t stride = gridDim.x * 4;
    for (; t < ntiles; t += stride) {
        const uint32_t ti = t / tiles_c, tj = t - ti * tiles_c;
        const uint32_t *s = src + ((int64_t)ti * 32 + c_in) * n + tj * 32 + 4 * q;
        uint32_t *d = dst + ((int64_t)ti * 32 + c_in) * n + tj * 32 + 4 * q;
        uint4 v[8];
#pragma unroll
        for (int g = 0; g < 8; ++g) v[g] = rapk::ldg_stream128(s + (int64_t)4 * g * n);
#pragma unroll
        for (int g = 0; g < 8; ++g) *reinterpret_cast<uint4 *>(d + (int64_t)4 * g * n) = v[g];
    }
}

// transpose without shared memory: 32-bit loads of a column run, 32-bit stores of a row run
__global__ void __launch_bounds__(128) regtranspose_kernel(const uint32_t *__restrict__ src, uint32_t *__restrict__ dst,
                                                           int64_t n, uint32_t tiles_c, uint32_t ntiles) {
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    uint32_t t = blockIdx.x * 4 + warp;
    const uint32_t stride = gridDim.x * 4;
    for (; t < ntiles; t += stride) {
        const uint32_t ti = t / tiles_c, tj = t - ti * tiles_c;
        // lane reads row r0+lane? no: coalesced read of row r, lanes = columns; 32 rows
        uint32_t v[32];
#pragma unroll
        for (int r = 0; r < 32; ++r) v[r] = __ldg(src + ((int64_t)ti * 32 + r) * n + tj * 32 + lane);
        // lane holds column (tj*32+lane) of rows r0..r0+31 = output row (tj*32+lane), cols r0..
        uint4 *o = reinterpret_cast<uint4 *>(dst + ((int64_t)tj * 32 + lane) * n + ti * 32);
#pragma unroll
        for (int k = 0; k < 8; ++k) o[k] = make_uint4(v[4 * k], v[4 * k + 1], v[4 * k + 2], v[4 * k + 3]);
    }
}

// copy probe: each warp copies an RT-row x (4096/RT)-byte block, 8 x 512 B instructions
template <int RT>
__global__ void __launch_bounds__(128) aspect_copy_kernel(const uint32_t *__restrict__ src, uint32_t *__restrict__ dst,
                                                          int64_t n, uint32_t nblocks) {
    constexpr int WB = 4096 / RT;                   // bytes per block row
    constexpr int WW = WB / 4;                      // words per block row
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    const uint32_t bpr = (uint32_t)(n / WW);        // blocks per matrix row-band
    for (uint32_t t = blockIdx.x * 4 + warp; t < nblocks; t += gridDim.x * 4) {
        const uint32_t bi = t / bpr, bj = t - bi * bpr;
        const int64_t base = (int64_t)bi * RT * n + (int64_t)bj * WW;
        uint4 v[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            const int off = 512 * i + 16 * lane;
            const int r = off / WB, cw = (off % WB) / 4;
            v[i] = rapk::ldg_stream128(src + base + (int64_t)r * n + cw);
        }
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            const int off = 512 * i + 16 * lane;
            const int r = off / WB, cw = (off % WB) / 4;
            *reinterpret_cast<uint4 *>(dst + base + (int64_t)r * n + cw) = v[i];
        }
    }
}

template <int RT>
static void run_aspect(const uint32_t *a, uint32_t *b, cudaEvent_t e0, cudaEvent_t e1) {
    const int64_t n = 8192;
    const uint32_t nb = (uint32_t)(n * n * 4 / 4096);
    int occ; cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, aspect_copy_kernel<RT>, 128, 0);
    std::vector<float> ms;
    for (int i = 0; i < 23; ++i) {
        cudaEventRecord(e0); aspect_copy_kernel<RT><<<148 * occ, 128>>>(a, b, n, nb); cudaEventRecord(e1);
        cudaEventSynchronize(e1); float t; cudaEventElapsedTime(&t, e0, e1); if (i >= 3) ms.push_back(t);
    }
    std::sort(ms.begin(), ms.end());
    printf("probe copy %2d rows x %4d B per warp block: %.1f GB/s\n", RT, 4096 / RT, 2.0 * n * n * 4 / ms[ms.size() / 2] / 1e6);
}

// ---- streaming-copy probes: which store/load flavour reaches the copy roofline
__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint4 ld_ef(const void *ptr, uint64_t pol) {
    uint4 r;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(ptr), "l"(pol));
    return r;
}
__device__ __forceinline__ void st_ef(void *ptr, uint4 v, uint64_t pol) {
    asm volatile("st.global.L1::no_allocate.L2::cache_hint.v4.u32 [%0], {%1,%2,%3,%4}, %5;"
                 :: "l"(ptr), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w), "l"(pol) : "memory");
}
__device__ __forceinline__ void st_cs(void *ptr, uint4 v) {
    asm volatile("st.global.cs.v4.u32 [%0], {%1,%2,%3,%4};" :: "l"(ptr), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}

template <int MODE, int U>   // MODE 0 plain, 1 st.cs, 2 ld evict_first, 3 ld+st evict_first
__global__ void __launch_bounds__(128) stream_copy_kernel(const uint4 *__restrict__ src, uint4 *__restrict__ dst, size_t n16) {
    const uint64_t pol = policy_evict_first();
    const size_t per = (size_t)32 * U;
    const size_t nb = n16 / per;
    const uint32_t lane = threadIdx.x & 31u;
    for (size_t b = blockIdx.x * 4 + (threadIdx.x >> 5); b < nb; b += (size_t)gridDim.x * 4) {
        uint4 v[U];
#pragma unroll
        for (int i = 0; i < U; ++i) {
            const uint4 *p = src + b * per + i * 32 + lane;
            v[i] = (MODE >= 2) ? ld_ef(p, pol) : rapk::ldg_stream128(p);
        }
#pragma unroll
        for (int i = 0; i < U; ++i) {
            uint4 *p = dst + b * per + i * 32 + lane;
            if (MODE == 1) st_cs(p, v[i]);
            else if (MODE == 3) st_ef(p, v[i], pol);
            else *p = v[i];
        }
    }
}

template <int MODE, int U>
static void run_stream(const uint32_t *a, uint32_t *b, size_t bytes, cudaEvent_t e0, cudaEvent_t e1, int occ_override = 0) {
    int occ; cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, stream_copy_kernel<MODE, U>, 128, 0);
    if (occ_override) occ = occ_override;
    std::vector<float> ms;
    for (int i = 0; i < 23; ++i) {
        cudaEventRecord(e0);
        stream_copy_kernel<MODE, U><<<148 * occ, 128>>>((const uint4 *)a, (uint4 *)b, bytes / 16);
        cudaEventRecord(e1); cudaEventSynchronize(e1);
        float t; cudaEventElapsedTime(&t, e0, e1); if (i >= 3) ms.push_back(t);
    }
    std::sort(ms.begin(), ms.end());
    printf("probe stream copy mode=%d unroll=%2d occ=%2d %5zu MiB: %.1f GB/s\n", MODE, U, occ, bytes >> 20, 2.0 * bytes / ms[ms.size() / 2] / 1e6);
}

// 128-byte-chunk block transpose: matrix of 8192 rows x 256 chunks (128 B each) ->
// chunk (r, k) goes to (k*32 + r%32 ... ) i.e. rows of 32 chunks written as columns.
// MODE 0: sequential reads, scattered 128 B writes; MODE 1: scattered reads, sequential writes
template <int MODE>
__global__ void __launch_bounds__(128) chunk_scatter_kernel(const uint32_t *__restrict__ src, uint32_t *__restrict__ dst,
                                                            int64_t n, uint32_t ntiles) {
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    const uint32_t tiles_c = (uint32_t)(n / 32);
    const uint32_t q = lane & 7u, c_in = lane >> 3;
    for (uint32_t t = blockIdx.x * 4 + warp; t < ntiles; t += gridDim.x * 4) {
        const uint32_t ti = t / tiles_c, tj = t - ti * tiles_c;
        // "tile" = 32 x 128 B; sequential side: rows ti*32.. of chunk column tj (like a tile);
        // the other side: the same 32 chunks placed at output rows tj*32.., chunk column ti
        uint4 v[8];
#pragma unroll
        for (int g = 0; g < 8; ++g) {
            const int64_t r = (int64_t)ti * 32 + 4 * g + c_in;
            const int64_t rs = MODE == 0 ? r : (int64_t)tj * 32 + 4 * g + c_in;
            const int64_t cs = MODE == 0 ? (int64_t)tj * 32 : (int64_t)ti * 32;
            v[g] = rapk::ldg_stream128(src + rs * n + cs + 4 * q);
        }
#pragma unroll
        for (int g = 0; g < 8; ++g) {
            const int64_t rd = MODE == 0 ? (int64_t)tj * 32 + 4 * g + c_in : (int64_t)ti * 32 + 4 * g + c_in;
            const int64_t cd = MODE == 0 ? (int64_t)ti * 32 : (int64_t)tj * 32;
            *reinterpret_cast<uint4 *>(dst + rd * n + cd + 4 * q) = v[g];
        }
    }
}

// block-transpose access pattern at chunk granularity CB bytes: the matrix (8192 rows x 32 KiB)
// is cut into chunks of CB bytes; a warp moves a "tile" of 32 chunks = rows r..r+RW-1 of a chunk
// column; the destination puts chunk (row, k) at (k*... ) transposed block position.
// READS: 0 = sequential (tile rows), 1 = scattered;  WRITES: 0 = sequential, 1 = scattered.
template <int CB, int RS, int WS>
__global__ void __launch_bounds__(128) chunkx_kernel(const uint32_t *__restrict__ src, uint32_t *__restrict__ dst,
                                                     int64_t n) {
    constexpr int LPC = CB / 16;                 // lanes per chunk
    constexpr int CPI = 32 / LPC;                // chunks per instruction
    constexpr int NCH = 32;                      // chunks per warp tile (8 instructions... 4096 B)
    constexpr int INSTR = NCH / CPI * 0 + (NCH * CB) / 512;
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    const int64_t cpr = n * 4 / CB;              // chunks per matrix row
    // tile = NCH chunks: rows (tr*NCH + i), chunk column tc  (i = 0..NCH-1)
    const int64_t ntr = n / NCH, ntiles = ntr * cpr;
    const int64_t tlim = min(ntiles, (int64_t)(n * n * 4 / (NCH * CB)));
    for (int64_t t = blockIdx.x * 4 + warp; t < tlim; t += gridDim.x * 4) {
        const int64_t tr = t / cpr, tc = t - tr * cpr;
        // transposed position: swap the roles of (tr, tc) inside a square block grid
        const int64_t sq = min(ntr, cpr);
        const int64_t bt = (tr % sq), bc = (tc % sq);
        const int64_t xr = tr - bt + bc, xc = tc - bc + bt;
        uint4 v[INSTR];
#pragma unroll
        for (int k = 0; k < INSTR; ++k) {
            const int i = k * CPI + lane / LPC;                     // chunk in tile
            const int64_t R = RS ? (xr * NCH + i) : (tr * NCH + i), C = RS ? xc : tc;
            v[k] = rapk::ldg_stream128(src + R * n + C * (CB / 4) + (lane % LPC) * 4);
        }
#pragma unroll
        for (int k = 0; k < INSTR; ++k) {
            const int i = k * CPI + lane / LPC;
            const int64_t R = WS ? (xr * NCH + i) : (tr * NCH + i), C = WS ? xc : tc;
            *reinterpret_cast<uint4 *>(dst + R * n + C * (CB / 4) + (lane % LPC) * 4) = v[k];
        }
    }
}

template <int CB, int RS, int WS>
static void run_chunkx(const uint32_t *a, uint32_t *b, cudaEvent_t e0, cudaEvent_t e1, int occ) {
    std::vector<float> ms;
    for (int i = 0; i < 23; ++i) {
        cudaEventRecord(e0); chunkx_kernel<CB, RS, WS><<<148 * occ, 128>>>(a, b, 8192); cudaEventRecord(e1);
        cudaEventSynchronize(e1); float t; cudaEventElapsedTime(&t, e0, e1); if (i >= 3) ms.push_back(t);
    }
    std::sort(ms.begin(), ms.end());
    printf("probe chunkx CB=%4d reads %s writes %s occ %d: %.1f GB/s\n", CB, RS ? "scattered" : "seq      ",
           WS ? "scattered" : "seq      ", occ, 2.0 * 8192.0 * 8192 * 4 / ms[ms.size() / 2] / 1e6);
}

// tile copy with the transpose's store granularity: 32 x STG.32 (one 128 B row each) per tile
template <int STW>   // STW = 1: 32-bit stores (lane = column), 4: 128-bit stores (8 lanes per row)
__global__ void __launch_bounds__(128) tilecopy_st_kernel(const uint32_t *__restrict__ src, uint32_t *__restrict__ dst,
                                                          int64_t n, uint32_t tiles_c, uint32_t ntiles) {
    __shared__ uint32_t sm[4][32 * 32];
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    const uint32_t q = lane & 7u, c_in = lane >> 3;
    uint32_t *tile = sm[warp];
    for (uint32_t t = blockIdx.x * 4 + warp; t < ntiles; t += gridDim.x * 4) {
        const uint32_t ti = t / tiles_c, tj = t - ti * tiles_c;
        const uint32_t *s = src + ((int64_t)ti * 32 + c_in) * n + tj * 32 + 4 * q;
        uint4 v[8];
#pragma unroll
        for (int g = 0; g < 8; ++g) v[g] = rapk::ldg_stream128(s + (int64_t)4 * g * n);
#pragma unroll
        for (int g = 0; g < 8; ++g) *reinterpret_cast<uint4 *>(&tile[(4 * g + c_in) * 32 + 4 * q]) = v[g];
        __syncwarp();
        if (STW == 1) {
            uint32_t *o = dst + (int64_t)ti * 32 * n + tj * 32 + lane;
#pragma unroll
            for (int r = 0; r < 32; ++r) o[(int64_t)r * n] = tile[r * 32 + lane];
        } else {
            uint32_t *o = dst + ((int64_t)ti * 32 + c_in) * n + tj * 32 + 4 * q;
#pragma unroll
            for (int g = 0; g < 8; ++g)
                *reinterpret_cast<uint4 *>(o + (int64_t)4 * g * n) = *reinterpret_cast<uint4 *>(&tile[(4 * g + c_in) * 32 + 4 * q]);
        }
        __syncwarp();
    }
}

static float median(std::vector<float> v) { std::sort(v.begin(), v.end()); return v[v.size() / 2]; }

int main(int argc, char **argv) {
    const int64_t n32 = 8192, n64 = 16384;
    const size_t bytes32 = n32 * n32 * 4, bytes64 = n64 * n64 * 8;
    uint32_t *a, *b; unsigned long long *bad;
    CK(cudaMalloc(&a, bytes64)); CK(cudaMalloc(&b, bytes64)); CK(cudaMalloc(&bad, 8));
    fill<<<4096, 256>>>(a, bytes64 / 4, 7); CK(cudaDeviceSynchronize());
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    auto timeit = [&](auto fn, int reps) {
        for (int i = 0; i < 3; ++i) fn();
        std::vector<float> ms;
        for (int i = 0; i < reps; ++i) {
            cudaEventRecord(e0); fn(); cudaEventRecord(e1); cudaEventSynchronize(e1);
            float t; cudaEventElapsedTime(&t, e0, e1); ms.push_back(t);
        }
        return median(ms);
    };
    {
        float t = timeit([&] { cudaMemcpyAsync(b, a, bytes32, cudaMemcpyDeviceToDevice); }, 20);
        printf("memcpy d2d %zu MiB: %.1f GB/s\n", bytes32 >> 20, 2.0 * bytes32 / t / 1e6);
        t = timeit([&] { cudaMemcpyAsync(b, a, bytes64, cudaMemcpyDeviceToDevice); }, 10);
        printf("memcpy d2d %zu MiB: %.1f GB/s\n", bytes64 >> 20, 2.0 * bytes64 / t / 1e6);
    }
    if (argc > 1 && std::string(argv[1]) == "shapes") {
        // partition-camping probe: the same kernel at power-of-two and padded pitches
        struct Case { int64_t rows, cols, ld_src, ld_dst; };
        const Case cases[] = {{8192, 8192, 8192, 8192}, {8192, 8192, 8224, 8224}, {8192, 8192, 8192 + 4, 8192 + 4},
                              {8000, 8000, 8000, 8000}, {8064, 8064, 8064, 8064}, {7936, 8192, 8192, 7936},
                              {4096, 16384, 16384, 4096}, {16384, 4096, 4096, 16384}, {11585, 11585, 11588, 11588}};
        for (const Case &cs : cases) {
            for (int lay : {RAP_LAYOUT_RAP, RAP_LAYOUT_PAD}) {
                rapk::TransposeTuning tu = rapk::default_tuning(4);
                const double bytes = 2.0 * cs.rows * cs.cols * 4;
                float t = timeit([&] { rapk::launch_transpose_tuned(a, b, cs.rows, cs.cols, cs.ld_src, cs.ld_dst, 4, lay, 1, tu, 0); }, 30);
                CK(cudaGetLastError());
                printf("b32 %s rows=%lld cols=%lld ld_src=%lld ld_dst=%lld : %7.1f GB/s %8.1f us\n", lay == RAP_LAYOUT_RAP ? "rap" : "pad",
                       (long long)cs.rows, (long long)cs.cols, (long long)cs.ld_src, (long long)cs.ld_dst, bytes / t / 1e6, t * 1e3);
            }
        }
        {
            const int64_t n = 8192; const uint32_t tc = 256, nt = 65536;
            int occ; cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, tilecopy_kernel<1>, 128, 0);
            float t = timeit([&] { tilecopy_kernel<1><<<148 * occ, 128>>>(a, b, n, tc, nt); }, 30);
            printf("probe tilecopy (same tile loads, row stores, occ %d): %.1f GB/s\n", occ, 2.0 * n * n * 4 / t / 1e6);
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, regtranspose_kernel, 128, 0);
            t = timeit([&] { regtranspose_kernel<<<148 * occ, 128>>>(a, b, n, tc, nt); }, 30);
            run_aspect<32>(a, b, e0, e1); run_aspect<16>(a, b, e0, e1); run_aspect<8>(a, b, e0, e1);
            run_aspect<4>(a, b, e0, e1); run_aspect<2>(a, b, e0, e1); run_aspect<1>(a, b, e0, e1);
            for (int o : {3, 4, 6, 8, 12, 16}) {
                float t1 = timeit([&] { tilecopy_st_kernel<1><<<148 * o, 128>>>(a, b, n, tc, nt); }, 30);
                float t4 = timeit([&] { tilecopy_st_kernel<4><<<148 * o, 128>>>(a, b, n, tc, nt); }, 30);
                printf("probe smem tilecopy occ %2d: STG.32 rows %.1f GB/s   STG.128 %.1f GB/s\n", o,
                       2.0 * n * n * 4 / t1 / 1e6, 2.0 * n * n * 4 / t4 / 1e6);
            }
            for (int o : {4, 6, 8}) {
                run_chunkx<128, 0, 0>(a, b, e0, e1, o); run_chunkx<128, 0, 1>(a, b, e0, e1, o); run_chunkx<128, 1, 1>(a, b, e0, e1, o);
                run_chunkx<256, 0, 0>(a, b, e0, e1, o); run_chunkx<256, 0, 1>(a, b, e0, e1, o); run_chunkx<256, 1, 1>(a, b, e0, e1, o);
                run_chunkx<512, 0, 0>(a, b, e0, e1, o); run_chunkx<512, 0, 1>(a, b, e0, e1, o); run_chunkx<512, 1, 1>(a, b, e0, e1, o);
            }
            for (int o : {2, 3, 4, 6, 8, 16}) {
                float t = timeit([&] { tilecopy_kernel<1><<<148 * o, 128>>>(a, b, n, tc, nt); }, 30);
                printf("probe tilecopy occ %2d: %.1f GB/s\n", o, 2.0 * n * n * 4 / t / 1e6);
                t = timeit([&] { chunk_scatter_kernel<0><<<148 * o, 128>>>(a, b, n, nt); }, 30);
                printf("probe chunk-transpose copy, seq reads / scattered 128B writes, occ %2d: %.1f GB/s\n", o, 2.0 * n * n * 4 / t / 1e6);
                t = timeit([&] { chunk_scatter_kernel<1><<<148 * o, 128>>>(a, b, n, nt); }, 30);
                printf("probe chunk-transpose copy, scattered reads / seq writes, occ %2d: %.1f GB/s\n", o, 2.0 * n * n * 4 / t / 1e6);
            }
            printf("probe register transpose (32-bit row loads, 128-bit uncoalesced-row stores, occ %d): %.1f GB/s\n", occ, 2.0 * n * n * 4 / t / 1e6);
        }
        for (size_t mb : {64, 128, 256, 512, 1024}) {
            size_t by = mb << 20;
            float t = timeit([&] { cudaMemcpyAsync(b, a, by, cudaMemcpyDeviceToDevice); }, 20);
            printf("memcpy d2d %zu MiB: %.1f GB/s\n", mb, 2.0 * by / t / 1e6);
        }
        return 0;
    }
    const int layouts[] = {RAP_LAYOUT_RAP, RAP_LAYOUT_RAW, RAP_LAYOUT_PAD, RAP_LAYOUT_XOR, RAP_LAYOUT_RAS};
    const char *lname[] = {"raw", "pad", "xor", "ras", "rap"};
    struct Shape { int depth, minb; bool vst; int sr, sc; bool tma; };
    const Shape shapes[] = {{1, 1, false, 8, 2, false}, {1, 1, false, 12, 1, false}, {1, 1, false, 4, 1, false}};
    for (int eb : {4, 8}) {
        const int64_t n = eb == 4 ? n32 : n64;
        const size_t bytes = eb == 4 ? bytes32 : bytes64;
        for (int lay : {RAP_LAYOUT_RAP, RAP_LAYOUT_RAW, RAP_LAYOUT_PAD, RAP_LAYOUT_XOR, RAP_LAYOUT_RAS}) {
            for (const Shape &sh : shapes) {
                if (lay != RAP_LAYOUT_RAP) continue;
                const int rp = (lay == RAP_LAYOUT_RAP || lay == RAP_LAYOUT_RAS) ? 64 : (lay == RAP_LAYOUT_PAD ? 33 : 32);
                if ((size_t)32 * rp * (eb / 4) * 4 * sh.sr * sh.sc + (sh.tma ? (size_t)1024 * eb * sh.sr * sh.sc : 0)
                    > 227 * 1024) continue;   // smem limit
                for (int cps : {0}) {
                    if (lay != RAP_LAYOUT_RAP && cps) continue;
                    rapk::TransposeTuning tu; tu.minb = sh.minb; tu.depth = sh.depth; tu.ctas_per_sm = cps;
                    tu.vst = sh.vst; tu.sr = sh.sr; tu.sc = sh.sc; tu.tma_store = sh.tma;
                    CK(cudaMemset(b, 0, bytes));
                    float t = timeit([&] { rapk::launch_transpose_tuned(a, b, n, n, n, n, eb, lay, 1, tu, 0); }, eb == 4 ? 30 : 10);
                    CK(cudaGetLastError());
                    CK(cudaMemset(bad, 0, 8));
                    check_t<<<2048, 256>>>(a, b, n, eb / 4, bad);
                    unsigned long long hb; CK(cudaMemcpy(&hb, bad, 8, cudaMemcpyDeviceToHost));
                    printf("b%d %-4s depth=%d minb=%d vst=%d tma=%d sr=%2d sc=%d ctas/sm=%d : %7.1f GB/s  %8.1f us  %s\n", eb * 8,
                           lname[lay], sh.depth, sh.minb, (int)sh.vst, (int)sh.tma, sh.sr, sh.sc, cps, 2.0 * bytes / t / 1e6, t * 1e3,
                           hb ? "MISMATCH" : "ok");
                }
            }
        }
    }
    return 0;
}
