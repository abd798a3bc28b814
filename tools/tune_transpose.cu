// tune_transpose.cu -- dev harness: times the transpose kernels of librap under launch-shape
// variants (register budget via __launch_bounds__ min blocks, tile traversal group) on the
// BASELINE cfg3 / cfg4 matrices, next to a device-to-device memcpy of the same bytes.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 \
//          -Ipaper_conf_icppw_nakanomi14_b200/csrc -o tools/tune_transpose tools/tune_transpose.cu
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <algorithm>
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
    const int layouts[] = {RAP_LAYOUT_RAP, RAP_LAYOUT_RAW, RAP_LAYOUT_PAD, RAP_LAYOUT_XOR};
    const char *lname[] = {"raw", "pad", "xor", "ras", "rap"};
    const int minbs[] = {1, 2, 3, 4};
    const uint32_t groups[] = {0, 8, 16, 32, 48, 64, 128};
    for (int eb : {4, 8}) {
        const int64_t n = eb == 4 ? n32 : n64;
        const size_t bytes = eb == 4 ? bytes32 : bytes64;
        for (int lay : layouts) {
            for (int mb : minbs) {
                if (lay != RAP_LAYOUT_RAP && mb != 2) continue;
                for (uint32_t g : groups) {
                    if (lay != RAP_LAYOUT_RAP && g != 0 && g != 32) continue;
                    rapk::TransposeTuning tu; tu.group = g; tu.minb = mb;
                    CK(cudaMemset(b, 0, bytes));
                    float t = timeit([&] { rapk::launch_transpose_tuned(a, b, n, n, n, n, eb, lay, 1, tu, 0); }, eb == 4 ? 30 : 10);
                    CK(cudaGetLastError());
                    CK(cudaMemset(bad, 0, 8));
                    check_t<<<2048, 256>>>(a, b, n, eb / 4, bad);
                    unsigned long long hb; CK(cudaMemcpy(&hb, bad, 8, cudaMemcpyDeviceToHost));
                    printf("b%d %-4s minb=%d group=%3u : %7.1f GB/s  %8.1f us  %s\n", eb * 8, lname[lay], mb, g,
                           2.0 * bytes / t / 1e6, t * 1e3, hb ? "MISMATCH" : "ok");
                }
            }
        }
    }
    return 0;
}
