// rap_rng.cuh -- device-side random draws of the RAP hot path (steps T0 / C1 / C2).
//
// Counter contract (include/rap.h; reading vi -- the paper only says P is
// "selected from all w! permutations uniformly at random", §IV):
//   word(seed, n, d, t) = Philox4x32-10(ctr = (n_lo, n_hi, t>>2, d), key = (seed_lo, seed_hi))[t&3]
// Warp-cooperative: lane l of a warp ends up holding P[l] (or r[l]), so a permutation is
// never materialised in memory -- it lives in one register per lane and is read by shuffle.
#pragma once
#include <stdint.h>

namespace rapk {

constexpr unsigned kFull = 0xffffffffu;
constexpr uint32_t kDomainFY = 0, kDomainRAS = 1, kDomainRandom = 2;

// high word of the 64-bit product (UMULHI on the device); the host build serves rap_perm_gen
// and the launch-time shift vectors of the transposes (the same functions, not a second copy)
__host__ __device__ __forceinline__ uint32_t umulhi32(uint32_t a, uint32_t b) {
#ifdef __CUDA_ARCH__
    return __umulhi(a, b);
#else
    return (uint32_t)(((uint64_t)a * b) >> 32);
#endif
}

__host__ __device__ __forceinline__ uint4 philox4x32_10(uint4 c, uint32_t k0, uint32_t k1) {
#pragma unroll
    for (int round = 0; round < 10; ++round) {
        if (round) { k0 += 0x9E3779B9u; k1 += 0xBB67AE85u; }
        const uint32_t lo0 = 0xD2511F53u * c.x, hi0 = umulhi32(0xD2511F53u, c.x);
        const uint32_t lo1 = 0xCD9E8D57u * c.z, hi1 = umulhi32(0xCD9E8D57u, c.z);
        c = make_uint4(hi1 ^ c.y ^ k0, lo1, hi0 ^ c.w ^ k1, lo0);
    }
    return c;
}

// The 4 words t = 4*blk .. 4*blk+3 of domain d for index n.
__host__ __device__ __forceinline__ uint4 philox_block(uint64_t seed, uint64_t n, uint32_t d, uint32_t blk) {
    return philox4x32_10(make_uint4((uint32_t)n, (uint32_t)(n >> 32), blk, d),
                         (uint32_t)seed, (uint32_t)(seed >> 32));
}

__host__ __device__ __forceinline__ uint32_t pick(uint4 v, uint32_t k) {
    uint32_t x = v.x;
    x = (k == 1) ? v.y : x;
    x = (k == 2) ? v.z : x;
    x = (k == 3) ? v.w : x;
    return x;
}

// one word, word(seed, n, d, t), computed on its own (random access into the stream)
__device__ __forceinline__ uint32_t word_at(uint64_t seed, uint64_t n, uint32_t d, uint32_t t) {
    return pick(philox_block(seed, n, d, t >> 2), t & 3u);
}

// floor(u * m / 2^32)
__host__ __device__ __forceinline__ uint32_t mulshift(uint32_t u, uint32_t m) { return umulhi32(u, m); }

// Serial form of T0 (one thread / the host): a = perm(seed, n, w), 2 <= w <= 256, Durstenfeld
// for k = w-1 .. 1 with j = floor(word(0, w-1-k) * (k+1) / 2^32), swap a[k], a[j].
__host__ __device__ inline void perm_serial(uint64_t seed, uint64_t n, uint32_t w, uint32_t *a) {
    for (uint32_t k = 0; k < w; ++k) a[k] = k;
    uint4 blk = make_uint4(0u, 0u, 0u, 0u);
    for (uint32_t t = 0; t + 1 < w; ++t) {
        if ((t & 3u) == 0) blk = philox_block(seed, n, kDomainFY, t >> 2);
        const uint32_t k = w - 1 - t;
        const uint32_t j = mulshift(pick(blk, t & 3u), k + 1);
        const uint32_t x = a[k];
        a[k] = a[j];
        a[j] = x;
    }
}

// Serial RAS shifts r[i] = floor(word(1, i) * w / 2^32), i < w.
__host__ __device__ inline void ras_serial(uint64_t seed, uint64_t n, uint32_t w, uint32_t *r) {
    uint4 blk = make_uint4(0u, 0u, 0u, 0u);
    for (uint32_t i = 0; i < w; ++i) {
        if ((i & 3u) == 0) blk = philox_block(seed, n, kDomainRAS, i >> 2);
        r[i] = mulshift(pick(blk, i & 3u), w);
    }
}

// word(seed, n, d, t) for t = lane: each of the first ceil(w/4) lanes computes one Philox
// block, every lane then picks its word with 4 shuffles.
__device__ __forceinline__ uint32_t lane_word(uint64_t seed, uint64_t n, uint32_t d, uint32_t lane) {
    const uint4 blk = philox_block(seed, n, d, lane);           // lanes >= 8 compute spare blocks
    const uint32_t src = lane >> 2;
    uint4 v;
    v.x = __shfl_sync(kFull, blk.x, src);
    v.y = __shfl_sync(kFull, blk.y, src);
    v.z = __shfl_sync(kFull, blk.z, src);
    v.w = __shfl_sync(kFull, blk.w, src);
    return pick(v, lane & 3);
}

// Durstenfeld shuffle on a warp (T0 / C2): given u = word(seed, n, 0, lane) in every lane,
// returns P[lane] for lane < w (lanes >= w return their own index).  For k = w-1 .. 1:
// j = floor(word(0, w-1-k) * (k+1) / 2^32) and a[k] <-> a[j]; lane l holds a[l], the swap is
// one shuffle with a per-lane source.
template <int W>
__device__ __forceinline__ uint32_t warp_fisher_yates(uint32_t u, uint32_t lane, uint32_t w_rt) {
    const uint32_t w = W ? (uint32_t)W : w_rt;
    uint32_t a = lane;
    // lane t precomputes j for step k = w-1-t, (k+1) = w-t
    const uint32_t jv = (lane + 1 < w) ? mulshift(u, w - lane) : 0u;
    if (W) {
#pragma unroll
        for (int t = 0; t < (W ? W - 1 : 1); ++t) {
            const uint32_t k = (uint32_t)(W - 1 - t);
            const uint32_t j = __shfl_sync(kFull, jv, t);
            const uint32_t src = (lane == k) ? j : ((lane == j) ? k : lane);
            a = __shfl_sync(kFull, a, src);
        }
    } else {
        for (uint32_t t = 0; t + 1 < w; ++t) {
            const uint32_t k = w - 1 - t;
            const uint32_t j = __shfl_sync(kFull, jv, t);
            const uint32_t src = (lane == k) ? j : ((lane == j) ? k : lane);
            a = __shfl_sync(kFull, a, src);
        }
    }
    return a;
}

// P[lane] = perm(seed, n, w)[lane]
template <int W>
__device__ __forceinline__ uint32_t warp_perm(uint64_t seed, uint64_t n, uint32_t lane, uint32_t w_rt) {
    return warp_fisher_yates<W>(lane_word(seed, n, kDomainFY, lane), lane, w_rt);
}

// r[lane] = floor(word(1, lane) * w / 2^32)
__device__ __forceinline__ uint32_t warp_ras_shift(uint64_t seed, uint64_t n, uint32_t lane, uint32_t w) {
    return mulshift(lane_word(seed, n, kDomainRAS, lane), w);
}

}  // namespace rapk
