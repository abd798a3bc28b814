// probe_cpasync.cu -- dev probe: RAP transpose with cp.async (LDGSTS) staging straight into the
// RAP-addressed tile (no register round trip), a ring of ST tile buffers per warp, against the
// library's LDG -> STS kernel on the same 8192^2 fp32 matrix.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -lineinfo \
//          -Ipaper_conf_icppw_nakanomi14_b200/csrc -o tools/probe_cpasync tools/probe_cpasync.cu
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <algorithm>
#include <string>
#include <functional>
#include "transpose.cu"

namespace rapk {  // the RAP-16 kernel lives in another translation unit; not probed here
cudaError_t launch_transpose_rap16(const void *, void *, int64_t, int64_t, int64_t, int64_t, uint64_t, cudaStream_t) {
    return cudaErrorNotSupported;
}
}  // namespace rapk

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e), __LINE__); exit(1);} } while (0)

__global__ void fill(uint32_t *p, size_t n, uint32_t salt) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
        uint32_t x = (uint32_t)i * 2654435761u ^ salt ^ (uint32_t)(i >> 32);
        x ^= x >> 16; x *= 0x7feb352du; x ^= x >> 15; x *= 0x846ca68bu; x ^= x >> 16;
        p[i] = x;
    }
}
__global__ void check_t(const uint32_t *a, const uint32_t *b, int64_t n, unsigned long long *bad) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n * n; i += (int64_t)gridDim.x * blockDim.x) {
        int64_t r = i / n, c = i % n;
        if (a[r * n + c] != b[c * n + r]) { atomicAdd(bad, 1ull); return; }
    }
}

__device__ __forceinline__ void cpa4(uint32_t saddr, const void *g) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" :: "r"(saddr), "l"(g) : "memory");
}
__device__ __forceinline__ void cpa_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cpa_wait() { asm volatile("cp.async.wait_group %0;" :: "n"(N) : "memory"); }

// MODE 0: wrapped rows (32 words, bank (j+P[i]) mod 32 via &31); 1: unwrapped 64-word rows
template <int SR, int SC, int ST, bool LOCK, int MODE>
__global__ void __launch_bounds__(SR * SC * 32, 1)
cpa_kernel(const uint32_t *__restrict__ src, uint32_t *__restrict__ dst, int64_t n, uint64_t seed,
           uint32_t tiles) {
    constexpr int RP = MODE == 0 ? 32 : 64;
    constexpr int TW = 32 * RP;                        // words per tile buffer
    extern __shared__ __align__(16) uint32_t sm[];
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    uint32_t *ring = sm + warp * ST * TW;
    const uint32_t ring_s = (uint32_t)__cvta_generic_to_shared(ring);
    const uint32_t P = rapk::warp_perm<32>(seed, 0, lane, 32);
    uint32_t soff[32];
#pragma unroll
    for (int i = 0; i < 32; ++i) {
        const uint32_t p = __shfl_sync(0xffffffffu, P, i);
        soff[i] = 4u * (MODE == 0 ? (i * RP + ((lane + p) & 31u)) : (i * RP + lane + p));
    }
    uint32_t goff[32];                                 // byte offsets of the 32 tile rows (< 4 GiB)
#pragma unroll
    for (int i = 0; i < 32; ++i) goff[i] = (uint32_t)(i * n * 4);
    const uint32_t drow = lane * RP;
    const uint32_t stc = tiles / SC, nst = (tiles / SR) * stc;
    const uint32_t wr = warp % SR, wc = warp / SR;
    auto issue = [&](uint32_t st, uint32_t buf) {
        if (st < nst) {
            const uint32_t si = st / stc, sj = st - si * stc;
            const int64_t r0 = (int64_t)(si * SR + wr) * 32, c0 = (int64_t)(sj * SC + wc) * 32;
            const char *g = reinterpret_cast<const char *>(src + r0 * n + c0 + lane);
            const uint32_t b = ring_s + buf * TW * 4;
#pragma unroll
            for (int i = 0; i < 32; ++i) cpa4(b + soff[i], g + goff[i]);
        }
        cpa_commit();
    };
    uint32_t st = blockIdx.x;
#pragma unroll
    for (int s = 0; s < ST - 1; ++s) issue(st + s * gridDim.x, s);
    for (uint32_t k = 0; st < nst; ++k, st += gridDim.x) {
        issue(st + (ST - 1) * gridDim.x, (k + ST - 1) % ST);
        cpa_wait<ST - 1>();
        __syncwarp();
        if (LOCK) __syncthreads();
        const uint32_t si = st / stc, sj = st - si * stc;
        const int64_t r0 = (int64_t)(si * SR + wr) * 32, c0 = (int64_t)(sj * SC + wc) * 32;
        const uint32_t *t = ring + (k % ST) * TW + drow;
        uint32_t *o = dst + c0 * n + r0 + lane;
#pragma unroll
        for (int c = 0; c < 32; ++c) {
            const uint32_t v = MODE == 0 ? t[(c + P) & 31u] : t[c + P];
            o[(int64_t)c * n] = v;
        }
        __syncwarp();
    }
    cpa_wait<0>();
}

// The library's LDG.128 -> STS.32 design with WRAPPED 32-word RAP rows (bank = address mod 32 =
// (j + P[i]) mod 32 with an explicit & 31), i.e. 4 KiB per tile: twice the warps per SM for the
// same shared memory, so super-tiles of up to 32 warps fit.
template <int SR, int SC, int MINB>
__global__ void __launch_bounds__(SR * SC * 32, MINB)
wrap_kernel(const uint32_t *__restrict__ src, uint32_t *__restrict__ dst, int64_t n, uint64_t seed,
            uint32_t tiles) {
    extern __shared__ __align__(16) uint32_t sm[];
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    uint32_t *tile = sm + warp * 1024;
    const uint32_t P = rapk::warp_perm<32>(seed, 0, lane, 32);
    tile[P] = lane;
    __syncwarp();
    const uint32_t pinv = tile[lane];
    __syncwarp();
    const uint32_t q = lane & 7u, c_in = lane >> 3;
    uint32_t row_g[8], rot_g[8];
#pragma unroll
    for (int g = 0; g < 8; ++g) {
        const uint32_t rr = 4 * g + c_in;                    // P value of the row this lane loads
        row_g[g] = __shfl_sync(0xffffffffu, pinv, rr);
        rot_g[g] = 4 * q + rr;                               // (4q + P[row]) ; & 31 per element
    }
    const uint32_t stc = tiles / SC, nst = (tiles / SR) * stc;
    const uint32_t wr = warp % SR, wc = warp / SR;
    auto load = [&](uint4 (&v)[8], uint32_t st) {
        const uint32_t si = st / stc, sj = st - si * stc;
        const int64_t r0 = (int64_t)(si * SR + wr) * 32, c0 = (int64_t)(sj * SC + wc) * 32;
        const uint32_t *base = src + r0 * n + c0 + 4 * q;
#pragma unroll
        for (int g = 0; g < 8; ++g) v[g] = rapk::ldg_stream128(base + (int64_t)row_g[g] * n);
    };
    uint32_t st = blockIdx.x;
    uint4 v[8];
    if (st < nst) load(v, st);
    while (st < nst) {
        const uint32_t cst = st;
        // opaque copies: keep the compiler from hoisting 64 tile-invariant smem addresses into
        // registers (they are recomputed per tile: 2 ALU ops per access)
        uint32_t Pv, rg[8];
        int64_t nv;
        asm volatile("mov.u32 %0, %1;" : "=r"(Pv) : "r"(P));
        asm volatile("mov.b64 %0, %1;" : "=l"(nv) : "l"(n));
#pragma unroll
        for (int g = 0; g < 8; ++g) asm volatile("mov.u32 %0, %1;" : "=r"(rg[g]) : "r"(rot_g[g]));
#pragma unroll
        for (int g = 0; g < 8; ++g) {
            const uint32_t w4[4] = {v[g].x, v[g].y, v[g].z, v[g].w};
#pragma unroll
            for (int k = 0; k < 4; ++k) tile[(row_g[g] << 5) | ((rg[g] + k) & 31u)] = w4[k];
        }
        __syncwarp();
        st += gridDim.x;
        if (st < nst) load(v, st);
        if (SR * SC > 1) __syncthreads();
        const uint32_t si = cst / stc, sj = cst - si * stc;
        const int64_t r0 = (int64_t)(si * SR + wr) * 32, c0 = (int64_t)(sj * SC + wc) * 32;
        uint32_t *o = dst + c0 * n + r0 + lane;
        const uint32_t rb = lane << 5;
#pragma unroll
        for (int c = 0; c < 32; ++c) {
            *o = tile[rb | ((Pv + c) & 31u)];
            o += nv;
        }
        __syncwarp();
    }
}

// The library's design (unwrapped 64-word RAP rows, LDG.128 -> STS.32 in P-residue groups,
// lockstep drains) with the lockstep widened across a thread-block cluster of CL CTAs stacked
// along the input rows: a cluster super-tile is (CL*SR) x SC tiles, drained behind one cluster
// barrier, so each output row receives CL*SR*128 B at once.
__device__ __forceinline__ void st_cs32(uint32_t *p, uint32_t v) {
    asm volatile("st.global.cs.u32 [%0], %1;" :: "l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void st_ef32(uint32_t *p, uint32_t v, uint64_t pol) {
    asm volatile("st.global.L2::cache_hint.u32 [%0], %1, %2;" :: "l"(p), "r"(v), "l"(pol) : "memory");
}
__device__ __forceinline__ uint4 ld_hint128(const void *p, uint64_t pol) {
    uint4 r;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p), "l"(pol));
    return r;
}

// ST: 0 plain stores, 1 st.global.cs, 2 L2 evict_first stores, 3 evict_first loads + stores,
//     4 evict_last stores (keep output lines in L2 so write-back happens in larger batches)
// GR > 1: cluster super-tiles visited in groups of GR super-tile rows (column-major inside a
// group), so the concurrently active clusters cover a squarish block of the matrix: shorter
// scattered write runs across output rows, more input rows read in parallel.
template <int SR, int SC, int CL, int ST = 0, int GR = 1>
__global__ void __launch_bounds__(SR * SC * 32, 1)
clu_kernel(const uint32_t *__restrict__ src, uint32_t *__restrict__ dst, int64_t n, uint64_t seed,
           uint32_t tiles) {
    extern __shared__ __align__(16) uint32_t sm[];
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    uint32_t *tile = sm + warp * 2048;
    const uint32_t P = rapk::warp_perm<32>(seed, 0, lane, 32);
    tile[P] = lane;
    __syncwarp();
    const uint32_t pinv = tile[lane];
    __syncwarp();
    const uint32_t q = lane & 7u, c_in = lane >> 3;
    uint32_t row_g[8], a_g[8];
#pragma unroll
    for (int g = 0; g < 8; ++g) {
        const uint32_t rr = 4 * g + c_in;
        row_g[g] = __shfl_sync(0xffffffffu, pinv, rr);
        a_g[g] = row_g[g] * 64 + 4 * q + rr;
    }
    const uint32_t drain_base = lane * 64 + P;
    uint64_t pol_ef, pol_el;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol_ef));
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol_el));
    uint32_t crank = 0, cid = blockIdx.x, ncl = gridDim.x;
    if (CL > 1) {
        asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(crank));
        asm volatile("mov.u32 %0, %%clusterid.x;" : "=r"(cid));
        asm volatile("mov.u32 %0, %%nclusterid.x;" : "=r"(ncl));
    }
    const uint32_t stc = tiles / SC, nst = (tiles / (SR * CL)) * stc;
    const uint32_t wr = crank * SR + warp % SR, wc = warp / SR;
    auto split = [&](uint32_t st, uint32_t &si, uint32_t &sj) {
        if (GR == 1) { si = st / stc; sj = st - si * stc; return; }
        const uint32_t g = st / (GR * stc), idx = st - g * (GR * stc);
        si = g * GR + idx % GR; sj = idx / GR;
    };
    auto load = [&](uint4 (&v)[8], uint32_t st) {
        uint32_t si, sj; split(st, si, sj);
        const int64_t r0 = (int64_t)(si * SR * CL + wr) * 32, c0 = (int64_t)(sj * SC + wc) * 32;
        const uint32_t *base = src + r0 * n + c0 + 4 * q;
#pragma unroll
        for (int g = 0; g < 8; ++g)
            v[g] = (ST == 3) ? ld_hint128(base + (int64_t)row_g[g] * n, pol_ef) : rapk::ldg_stream128(base + (int64_t)row_g[g] * n);
    };
    uint32_t st = cid;
    uint4 v[8];
    if (st < nst) load(v, st);
    while (st < nst) {
        const uint32_t cst = st;
#pragma unroll
        for (int g = 0; g < 8; ++g) {
            tile[a_g[g] + 0] = v[g].x; tile[a_g[g] + 1] = v[g].y;
            tile[a_g[g] + 2] = v[g].z; tile[a_g[g] + 3] = v[g].w;
        }
        __syncwarp();
        st += ncl;
        if (st < nst) load(v, st);
        if (CL > 1) {
            asm volatile("barrier.cluster.arrive.relaxed.aligned;" ::: "memory");
            asm volatile("barrier.cluster.wait.aligned;" ::: "memory");
        } else {
            __syncthreads();
        }
        uint32_t si, sj; split(cst, si, sj);
        const int64_t r0 = (int64_t)(si * SR * CL + wr) * 32, c0 = (int64_t)(sj * SC + wc) * 32;
        uint32_t *o = dst + c0 * n + r0 + lane;
#pragma unroll
        for (int c = 0; c < 32; ++c) {
            const uint32_t x = tile[drain_base + c];
            if (ST == 1) st_cs32(o, x);
            else if (ST == 2 || ST == 3) st_ef32(o, x, pol_ef);
            else if (ST == 4) st_ef32(o, x, pol_el);
            else *o = x;
            o += n;
        }
        __syncwarp();
    }
}


// K-plane fp32 tile: one warp owns a (32K) x 32 tile of 32-bit elements held as K RAP planes,
// plane p row i = input row K*i + p (each plane the paper's 32 x 32 RAP tile with the same P).
// The drain reads the K planes at the same (conflict-free, stride) address and writes K adjacent
// output columns with one K-word store: 64-/128-bit STG, 256 / 512 B per warp instruction per
// output row, and K x 4 KiB of loads in flight per warp.  RP = 64: unwrapped rows, 32: wrapped.
template <int K, int SR, int SC, int CL, int RP>
__global__ void __launch_bounds__(SR * SC * 32, 1)
kplane_kernel(const uint32_t *__restrict__ src, uint32_t *__restrict__ dst, int64_t n, uint64_t seed,
              uint32_t tiles) {
    constexpr int PW = 32 * RP;
    extern __shared__ __align__(16) uint32_t sm[];
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    uint32_t *tile = sm + warp * K * PW;
    const uint32_t P = rapk::warp_perm<32>(seed, 0, lane, 32);
    tile[P] = lane;
    __syncwarp();
    const uint32_t pinv = tile[lane];
    __syncwarp();
    const uint32_t q = lane & 7u, c_in = lane >> 3;
    uint32_t row_g[8], a_g[8];
#pragma unroll
    for (int g = 0; g < 8; ++g) {
        const uint32_t rr = 4 * g + c_in;            // = P[row_g[g]]
        row_g[g] = __shfl_sync(0xffffffffu, pinv, rr);
        a_g[g] = RP == 64 ? row_g[g] * 64 + 4 * q + rr : row_g[g] * 32;
    }
    uint32_t crank = 0, cid = blockIdx.x, ncl = gridDim.x;
    if (CL > 1) {
        asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(crank));
        asm volatile("mov.u32 %0, %%clusterid.x;" : "=r"(cid));
        asm volatile("mov.u32 %0, %%nclusterid.x;" : "=r"(ncl));
    }
    const uint32_t rtiles = tiles / K;
    const uint32_t stc = tiles / SC, nst = (rtiles / (SR * CL)) * stc;
    const uint32_t wr = crank * SR + warp % SR, wc = warp / SR;
    auto load = [&](uint4 (&v)[K][8], uint32_t st) {
        const uint32_t si = st / stc, sj = st - si * stc;
        const int64_t r0 = (int64_t)(si * SR * CL + wr) * 32 * K, c0 = (int64_t)(sj * SC + wc) * 32;
        const uint32_t *base = src + r0 * n + c0 + 4 * q;
#pragma unroll
        for (int p = 0; p < K; ++p)
#pragma unroll
            for (int g = 0; g < 8; ++g) v[p][g] = rapk::ldg_stream128(base + (int64_t)(K * row_g[g] + p) * n);
    };
    uint32_t st = cid;
    uint4 v[K][8];
    if (st < nst) load(v, st);
    while (st < nst) {
        const uint32_t cst = st;
#pragma unroll
        for (int p = 0; p < K; ++p)
#pragma unroll
            for (int g = 0; g < 8; ++g) {
                const uint32_t w4[4] = {v[p][g].x, v[p][g].y, v[p][g].z, v[p][g].w};
#pragma unroll
                for (int e = 0; e < 4; ++e) {
                    const uint32_t off = RP == 64 ? a_g[g] + e : a_g[g] + ((4 * q + e + 4 * g + c_in) & 31u);
                    tile[p * PW + off] = w4[e];
                }
            }
        __syncwarp();
        st += ncl;
        if (st < nst) load(v, st);
        if (CL > 1) {
            asm volatile("barrier.cluster.arrive.relaxed.aligned;" ::: "memory");
            asm volatile("barrier.cluster.wait.aligned;" ::: "memory");
        } else if (SR * SC > 1) {
            __syncthreads();
        }
        const uint32_t si = cst / stc, sj = cst - si * stc;
        const int64_t r0 = (int64_t)(si * SR * CL + wr) * 32 * K, c0 = (int64_t)(sj * SC + wc) * 32;
        uint32_t *o = dst + c0 * n + r0 + K * lane;
#pragma unroll
        for (int c = 0; c < 32; ++c) {
            const uint32_t off = RP == 64 ? lane * 64 + P + c : lane * 32 + ((P + c) & 31u);
            if (K == 2) *reinterpret_cast<uint2 *>(o) = make_uint2(tile[off], tile[PW + off]);
            else *reinterpret_cast<uint4 *>(o) = make_uint4(tile[off], tile[PW + off], tile[2 * PW + off], tile[3 * PW + off]);
            o += n;
        }
        __syncwarp();
    }
}


// Memory-level-parallelism variants of the cluster kernel: MINB CTAs per SM (register budget),
// DEPTH tiles of loads in flight per warp (1 or 2 register buffers), RP = 64 unwrapped / 32
// wrapped RAP rows (half the shared memory per warp).
template <int SR, int SC, int CL, int MINB, int DEPTH, int RP>
__global__ void __launch_bounds__(SR * SC * 32, MINB)
mlp_kernel(const uint32_t *__restrict__ src, uint32_t *__restrict__ dst, int64_t n, uint64_t seed,
           uint32_t tiles) {
    extern __shared__ __align__(16) uint32_t sm[];
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    uint32_t *tile = sm + warp * 32 * RP;
    const uint32_t P = rapk::warp_perm<32>(seed, 0, lane, 32);
    tile[P] = lane;
    __syncwarp();
    const uint32_t pinv = tile[lane];
    __syncwarp();
    const uint32_t q = lane & 7u, c_in = lane >> 3;
    uint32_t row_g[8], a_g[8];
#pragma unroll
    for (int g = 0; g < 8; ++g) {
        const uint32_t rr = 4 * g + c_in;
        row_g[g] = __shfl_sync(0xffffffffu, pinv, rr);
        a_g[g] = RP == 64 ? row_g[g] * 64 + 4 * q + rr : row_g[g] * 32;
    }
    uint32_t crank = 0, cid = blockIdx.x, ncl = gridDim.x;
    if (CL > 1) {
        asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(crank));
        asm volatile("mov.u32 %0, %%clusterid.x;" : "=r"(cid));
        asm volatile("mov.u32 %0, %%nclusterid.x;" : "=r"(ncl));
    }
    const uint32_t stc = tiles / SC, nst = (tiles / (SR * CL)) * stc;
    const uint32_t wr = crank * SR + warp % SR, wc = warp / SR;
    auto load = [&](uint4 (&v)[8], uint32_t st) {
        const uint32_t si = st / stc, sj = st - si * stc;
        const int64_t r0 = (int64_t)(si * SR * CL + wr) * 32, c0 = (int64_t)(sj * SC + wc) * 32;
        const uint32_t *base = src + r0 * n + c0 + 4 * q;
#pragma unroll
        for (int g = 0; g < 8; ++g) v[g] = rapk::ldg_stream128(base + (int64_t)row_g[g] * n);
    };
    auto store = [&](const uint4 (&v)[8]) {
#pragma unroll
        for (int g = 0; g < 8; ++g) {
            const uint32_t w4[4] = {v[g].x, v[g].y, v[g].z, v[g].w};
#pragma unroll
            for (int e = 0; e < 4; ++e)
                tile[RP == 64 ? a_g[g] + e : a_g[g] + ((4 * q + e + 4 * g + c_in) & 31u)] = w4[e];
        }
    };
    auto sync = [&]() {
        if (CL > 1) {
            asm volatile("barrier.cluster.arrive.relaxed.aligned;" ::: "memory");
            asm volatile("barrier.cluster.wait.aligned;" ::: "memory");
        } else if (SR * SC > 1) {
            __syncthreads();
        }
    };
    auto drain = [&](uint32_t cst) {
        const uint32_t si = cst / stc, sj = cst - si * stc;
        const int64_t r0 = (int64_t)(si * SR * CL + wr) * 32, c0 = (int64_t)(sj * SC + wc) * 32;
        uint32_t *o = dst + c0 * n + r0 + lane;
#pragma unroll
        for (int c = 0; c < 32; ++c) {
            *o = tile[RP == 64 ? lane * 64 + P + c : lane * 32 + ((P + c) & 31u)];
            o += n;
        }
    };
    uint32_t st = cid;
    if (DEPTH == 1) {
        uint4 v[8];
        if (st < nst) load(v, st);
        while (st < nst) {
            const uint32_t cst = st;
            store(v);
            __syncwarp();
            st += ncl;
            if (st < nst) load(v, st);
            sync();
            drain(cst);
            __syncwarp();
        }
    } else {
        uint4 va[8], vb[8];
        if (st < nst) load(va, st);
        if (st + ncl < nst) load(vb, st + ncl);
        while (st < nst) {
            store(va);
            __syncwarp();
            if (st + 2 * ncl < nst) load(va, st + 2 * ncl);
            sync();
            drain(st);
            __syncwarp();
            st += ncl;
            if (st >= nst) break;
            store(vb);
            __syncwarp();
            if (st + 2 * ncl < nst) load(vb, st + 2 * ncl);
            sync();
            drain(st);
            __syncwarp();
            st += ncl;
        }
    }
}

// Warp-specialised variant: T = SR*SC producer warps (LDG.128 -> STS.32 into the RAP tile, the
// next tile's loads in flight while waiting for a free stage) and T consumer warps (lockstep drain
// of the super-tile: LDS column reads + 128 B STG rows), two super-tile stages in shared memory,
// handed over with named barriers (FULL[s] = 1 + s, EMPTY[s] = 3 + s) instead of one CTA barrier.
__device__ __forceinline__ void nb_sync(int id, int n) { asm volatile("bar.sync %0, %1;" :: "r"(id), "r"(n) : "memory"); }
__device__ __forceinline__ void nb_arrive(int id, int n) { asm volatile("bar.arrive %0, %1;" :: "r"(id), "r"(n) : "memory"); }

template <int SR, int SC>
__global__ void __launch_bounds__(2 * SR * SC * 32, 1)
ws_kernel(const uint32_t *__restrict__ src, uint32_t *__restrict__ dst, int64_t n, uint64_t seed,
          uint32_t tiles) {
    constexpr int T = SR * SC, NT = 2 * T * 32;
    extern __shared__ __align__(16) uint32_t sm[];
    const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    const bool producer = warp < T;
    const uint32_t w = producer ? warp : warp - T;          // tile slot in the super-tile
    uint32_t *tile0 = sm + w * 2048, *tile1 = sm + (T + w) * 2048;
    const uint32_t P = rapk::warp_perm<32>(seed, 0, lane, 32);
    const uint32_t stc = tiles / SC, nst = (tiles / SR) * stc;
    const uint32_t wr = w % SR, wc = w / SR;
    if (producer) {
        tile0[P] = lane;
        __syncwarp();
        const uint32_t pinv = tile0[lane];
        __syncwarp();
        const uint32_t q = lane & 7u, c_in = lane >> 3;
        uint32_t row_g[8], a_g[8];
#pragma unroll
        for (int g = 0; g < 8; ++g) {
            const uint32_t rr = 4 * g + c_in;
            row_g[g] = __shfl_sync(0xffffffffu, pinv, rr);
            a_g[g] = row_g[g] * 64 + 4 * q + rr;
        }
        auto load = [&](uint4 (&v)[8], uint32_t st) {
            const uint32_t si = st / stc, sj = st - si * stc;
            const int64_t r0 = (int64_t)(si * SR + wr) * 32, c0 = (int64_t)(sj * SC + wc) * 32;
            const uint32_t *base = src + r0 * n + c0 + 4 * q;
#pragma unroll
            for (int g = 0; g < 8; ++g) v[g] = rapk::ldg_stream128(base + (int64_t)row_g[g] * n);
        };
        uint4 va[8], vb[8];
        uint32_t st = blockIdx.x, k = 0;
        if (st < nst) load(va, st);
        while (st < nst) {
            const uint32_t nx = st + gridDim.x;
            if (nx < nst) load(vb, nx);                      // next tile in flight
            uint32_t *t = (k & 1) ? tile1 : tile0;
            if (k >= 2) nb_sync(3 + (k & 1), NT);            // wait: stage drained
#pragma unroll
            for (int g = 0; g < 8; ++g) {
                t[a_g[g] + 0] = va[g].x; t[a_g[g] + 1] = va[g].y;
                t[a_g[g] + 2] = va[g].z; t[a_g[g] + 3] = va[g].w;
            }
            nb_arrive(1 + (k & 1), NT);                      // stage full
#pragma unroll
            for (int g = 0; g < 8; ++g) va[g] = vb[g];
            st = nx; ++k;
        }
    } else {
        const uint32_t drain_base = lane * 64 + P;
        uint32_t st = blockIdx.x, k = 0;
        while (st < nst) {
            const uint32_t *t = (k & 1) ? tile1 : tile0;
            nb_sync(1 + (k & 1), NT);                        // wait: stage full (all T tiles)
            const uint32_t si = st / stc, sj = st - si * stc;
            const int64_t r0 = (int64_t)(si * SR + wr) * 32, c0 = (int64_t)(sj * SC + wc) * 32;
            uint32_t *o = dst + c0 * n + r0 + lane;
#pragma unroll
            for (int c = 0; c < 32; ++c) {
                *o = t[drain_base + c];
                o += n;
            }
            nb_arrive(3 + (k & 1), NT);                      // stage free
            st += gridDim.x; ++k;
        }
    }
}

static float median(std::vector<float> v) { std::sort(v.begin(), v.end()); return v[v.size() / 2]; }

int main(int argc, char **argv) {
    const int64_t n = 8192;
    const size_t bytes = n * n * 4;
    uint32_t *a, *b; unsigned long long *bad;
    CK(cudaMalloc(&a, bytes)); CK(cudaMalloc(&b, bytes)); CK(cudaMalloc(&bad, 8));
    fill<<<4096, 256>>>(a, bytes / 4, 7); CK(cudaDeviceSynchronize());
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
    auto check = [&](const char *name, float t) {
        CK(cudaGetLastError());
        CK(cudaMemset(bad, 0, 8));
        check_t<<<2048, 256>>>(a, b, n, bad);
        unsigned long long hb; CK(cudaMemcpy(&hb, bad, 8, cudaMemcpyDeviceToHost));
        printf("%-44s: %7.1f GB/s %8.1f us %s\n", name, 2.0 * bytes / t / 1e6, t * 1e3, hb ? "MISMATCH" : "ok");
        CK(cudaMemset(b, 0, bytes));
    };
    {
        float t = timeit([&] { cudaMemcpyAsync(b, a, bytes, cudaMemcpyDeviceToDevice); }, 30);
        printf("memcpy d2d 256 MiB: %.1f GB/s\n", 2.0 * bytes / t / 1e6);
    }
    {
        rapk::TransposeTuning tu = rapk::default_tuning(4);
        float t = timeit([&] { rapk::launch_transpose_tuned(a, b, n, n, n, n, 4, RAP_LAYOUT_RAP, 1, tu, 0); }, 30);
        check("library rap (LDG->STS, 8x2, unwrapped)", t);
    }
#define RUN(SR, SC, ST, LOCK, MODE, CPS)                                                                     \
    {                                                                                                        \
        auto k = cpa_kernel<SR, SC, ST, LOCK, MODE>;                                                         \
        const size_t smem = (size_t)SR * SC * ST * 32 * (MODE == 0 ? 32 : 64) * 4;                           \
        if (smem <= 227 * 1024) {                                                                            \
            CK(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));            \
            int occ; CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k, SR * SC * 32, smem));        \
            if (CPS && CPS < occ) occ = CPS;                                                                 \
            const uint32_t nst = (uint32_t)((n / 32 / SR) * (n / 32 / SC));                                  \
            const uint32_t grid = std::min<uint32_t>(nst, 148u * occ);                                       \
            float t = timeit([&] { k<<<grid, SR * SC * 32, smem>>>(a, b, n, 1, (uint32_t)(n / 32)); }, 30);  \
            char nm[128]; snprintf(nm, sizeof nm, "cp.async sr=%d sc=%d st=%d lock=%d mode=%d occ=%d", SR, SC, ST, (int)LOCK, MODE, occ); \
            check(nm, t);                                                                                    \
        }                                                                                                    \
    }
#define WRUN(SR, SC, MINB)                                                                                   \
    {                                                                                                        \
        auto k = wrap_kernel<SR, SC, MINB>;                                                                  \
        const size_t smem = (size_t)SR * SC * 4096;                                                          \
        CK(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));                \
        int occ; CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k, SR * SC * 32, smem));            \
        const uint32_t nst = (uint32_t)((n / 32 / SR) * (n / 32 / SC));                                      \
        const uint32_t grid = std::min<uint32_t>(nst, 148u * occ);                                           \
        float t = timeit([&] { k<<<grid, SR * SC * 32, smem>>>(a, b, n, 1, (uint32_t)(n / 32)); }, 30);      \
        char nm[128]; snprintf(nm, sizeof nm, "wrapped sr=%d sc=%d minb=%d occ=%d", SR, SC, MINB, occ);      \
        check(nm, t);                                                                                        \
    }
    // A/B of the cluster-lockstep variants against the library kernel: every variant is timed in
    // each of R interleaved rounds (so clock / thermal drift hits all alike); median of rounds
    std::vector<std::pair<std::string, std::function<void()>>> vs;
    {
        rapk::TransposeTuning tu = rapk::default_tuning(4);
        vs.push_back({"library rap default (4x2 warps, cluster 4)",
                      [=] { rapk::launch_transpose_tuned(a, b, n, n, n, n, 4, RAP_LAYOUT_RAP, 1, tu, 0); }});
        rapk::TransposeTuning t1 = tu;
        t1.cl = 1;
        vs.push_back({"library rap 8x2, no cluster (round-1 default)",
                      [=] { rapk::launch_transpose_tuned(a, b, n, n, n, n, 4, RAP_LAYOUT_RAP, 1, t1, 0); }});
        for (int lay : {RAP_LAYOUT_RAW, RAP_LAYOUT_PAD, RAP_LAYOUT_XOR, RAP_LAYOUT_RAS}) {
            static const char *nm[] = {"raw", "pad", "xor", "ras"};
            vs.push_back({std::string("library default layout ") + nm[lay],
                          [=] { rapk::launch_transpose_tuned(a, b, n, n, n, n, 4, lay, 1, tu, 0); }});
        }
    }
    auto add_cluster = [&](auto k, int SR, int SC, int CL) {
        const size_t smem = (size_t)SR * SC * 8192;
        CK(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        if (CL > 1) CK(cudaFuncSetAttribute(k, cudaFuncAttributeNonPortableClusterSizeAllowed, 1));
        cudaLaunchConfig_t cfg = {};
        static cudaLaunchAttribute at[64][1];
        static int nat = 0;
        cudaLaunchAttribute *ap = at[nat++];
        ap[0].id = cudaLaunchAttributeClusterDimension;
        ap[0].val.clusterDim.x = CL; ap[0].val.clusterDim.y = 1; ap[0].val.clusterDim.z = 1;
        cfg.blockDim = dim3(SR * SC * 32); cfg.dynamicSmemBytes = smem; cfg.attrs = ap; cfg.numAttrs = 1;
        int ncl = 0;
        cfg.gridDim = dim3(148 * CL);
        CK(cudaOccupancyMaxActiveClusters(&ncl, k, &cfg));
        const uint32_t nst = (uint32_t)((n / 32 / (SR * CL)) * (n / 32 / SC));
        cfg.gridDim = dim3(std::min<uint32_t>(nst, (uint32_t)ncl) * CL);
        static int idx = 0;
        char nm[128]; snprintf(nm, sizeof nm, "cluster sr=%d sc=%d cl=%d clusters=%d #%d", SR, SC, CL, ncl, idx++);
        vs.push_back({nm, [=] { cudaLaunchKernelEx(&cfg, k, (const uint32_t *)a, b, n, (uint64_t)1, (uint32_t)(n / 32)); }});
    };
    auto add_kp = [&](auto k, int K, int SR, int SC, int CL, int RP) {
        const size_t smem = (size_t)SR * SC * K * 32 * RP * 4;
        CK(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        if (CL > 1) CK(cudaFuncSetAttribute(k, cudaFuncAttributeNonPortableClusterSizeAllowed, 1));
        cudaLaunchConfig_t cfg = {};
        static cudaLaunchAttribute at[64][1];
        static int nat = 0;
        cudaLaunchAttribute *ap = at[nat++];
        ap[0].id = cudaLaunchAttributeClusterDimension;
        ap[0].val.clusterDim.x = CL; ap[0].val.clusterDim.y = 1; ap[0].val.clusterDim.z = 1;
        cfg.blockDim = dim3(SR * SC * 32); cfg.dynamicSmemBytes = smem; cfg.attrs = ap; cfg.numAttrs = 1;
        int ncl = 0;
        cfg.gridDim = dim3(148 * CL);
        CK(cudaOccupancyMaxActiveClusters(&ncl, k, &cfg));
        const uint32_t nst = (uint32_t)((n / 32 / K / (SR * CL)) * (n / 32 / SC));
        cfg.gridDim = dim3(std::min<uint32_t>(nst, (uint32_t)ncl) * CL);
        static int idx = 0;
        char nm[128]; snprintf(nm, sizeof nm, "kplane K=%d sr=%d sc=%d cl=%d rp=%d clusters=%d #%d", K, SR, SC, CL, RP, ncl, idx++);
        vs.push_back({nm, [=] { cudaLaunchKernelEx(&cfg, k, (const uint32_t *)a, b, n, (uint64_t)1, (uint32_t)(n / 32)); }});
    };
    auto add_mlp = [&](auto k, int SR, int SC, int CL, int MINB, int DEPTH, int RP) {
        const size_t smem = (size_t)SR * SC * 32 * RP * 4;
        CK(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        if (CL > 1) CK(cudaFuncSetAttribute(k, cudaFuncAttributeNonPortableClusterSizeAllowed, 1));
        cudaLaunchConfig_t cfg = {};
        static cudaLaunchAttribute at[64][1];
        static int nat = 0;
        cudaLaunchAttribute *ap = at[nat++];
        ap[0].id = cudaLaunchAttributeClusterDimension;
        ap[0].val.clusterDim.x = CL; ap[0].val.clusterDim.y = 1; ap[0].val.clusterDim.z = 1;
        cfg.blockDim = dim3(SR * SC * 32); cfg.dynamicSmemBytes = smem; cfg.attrs = ap; cfg.numAttrs = 1;
        int ncl = 0;
        cfg.gridDim = dim3(148 * CL);
        CK(cudaOccupancyMaxActiveClusters(&ncl, k, &cfg));
        const uint32_t nst = (uint32_t)((n / 32 / (SR * CL)) * (n / 32 / SC));
        cfg.gridDim = dim3(std::min<uint32_t>(nst, (uint32_t)ncl) * CL);
        cudaFuncAttributes fa; cudaFuncGetAttributes(&fa, k);
        char nm[160]; snprintf(nm, sizeof nm, "mlp sr=%d sc=%d cl=%d minb=%d depth=%d rp=%d regs=%d clusters=%d", SR, SC, CL, MINB, DEPTH, RP, fa.numRegs, ncl);
        vs.push_back({nm, [=] { cudaLaunchKernelEx(&cfg, k, (const uint32_t *)a, b, n, (uint64_t)1, (uint32_t)(n / 32)); }});
    };
    // grid size: cluster counts that divide the 2048 cluster super-tiles evenly vs all co-resident
    auto add_grid = [&](int want) {
        auto k = mlp_kernel<4, 2, 4, 2, 1, 64>;
        const size_t smem = (size_t)8 * 32 * 64 * 4;
        CK(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        cudaLaunchConfig_t cfg = {};
        static cudaLaunchAttribute at[16][1];
        static int nat = 0;
        cudaLaunchAttribute *ap = at[nat++];
        ap[0].id = cudaLaunchAttributeClusterDimension;
        ap[0].val.clusterDim.x = 4; ap[0].val.clusterDim.y = 1; ap[0].val.clusterDim.z = 1;
        cfg.blockDim = dim3(256); cfg.dynamicSmemBytes = smem; cfg.attrs = ap; cfg.numAttrs = 1;
        int ncl = 0;
        cfg.gridDim = dim3(148 * 4);
        CK(cudaOccupancyMaxActiveClusters(&ncl, k, &cfg));
        const int use = want > 0 ? std::min(want, ncl) : ncl;
        cfg.gridDim = dim3(use * 4);
        char nm[128]; snprintf(nm, sizeof nm, "cluster 4x2x4 grid %d of %d clusters", use, ncl);
        vs.push_back({nm, [=] { cudaLaunchKernelEx(&cfg, k, (const uint32_t *)a, b, n, (uint64_t)1, (uint32_t)(n / 32)); }});
    };
    add_grid(0);
    add_grid(64);
    add_grid(68);
    add_grid(57);
    add_grid(32);
    auto add_ws = [&](auto k, int SR, int SC) {
        const size_t smem = (size_t)2 * SR * SC * 8192;
        CK(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        const uint32_t nst = (uint32_t)((n / 32 / SR) * (n / 32 / SC));
        int occ = 1;
        CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k, 2 * SR * SC * 32, smem));
        const uint32_t grid = std::min<uint32_t>(nst, 148u * occ);
        char nm[128]; snprintf(nm, sizeof nm, "warp-specialised sr=%d sc=%d (2 stages) occ=%d", SR, SC, occ);
        vs.push_back({nm, [=] { k<<<grid, 2 * SR * SC * 32, smem>>>(a, b, n, (uint64_t)1, (uint32_t)(n / 32)); }});
    };
    vs.push_back({"memcpy d2d 256 MiB", [=] { cudaMemcpyAsync(b, a, bytes, cudaMemcpyDeviceToDevice); }});
    const int R = argc > 1 ? atoi(argv[1]) : 7;
    std::vector<std::vector<float>> res(vs.size());
    for (int r = 0; r < R; ++r)
        for (size_t v = 0; v < vs.size(); ++v) res[v].push_back(timeit(vs[v].second, 20));
    for (size_t v = 0; v < vs.size(); ++v) {
        const float t = median(res[v]);
        if (vs[v].first.rfind("memcpy", 0) == 0) {
            printf("%-44s: %7.1f GB/s %8.1f us (median of %d rounds)\n", vs[v].first.c_str(), 2.0 * bytes / t / 1e6, t * 1e3, R);
            continue;
        }
        vs[v].second();
        check(vs[v].first.c_str(), t);
    }
    return 0;
}
