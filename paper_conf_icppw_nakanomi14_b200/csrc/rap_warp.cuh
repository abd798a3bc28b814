// rap_warp.cuh -- the warp-level DMM congestion primitives shared by the evaluator kernels
// (§II): one CUDA warp = one DMM warp of w <= 32 threads.
#pragma once
#include <stdint.h>

#include "rap_rng.cuh"

namespace rapk {

// ---------------------------------------------------------------------------------------
// Congestion by bit-sliced ballots (default).  Each lane v counts the requests to bank v:
// with B_k = ballot(bit k of bank), the lanes whose bank equals v are AND_k (v_k ? B_k : ~B_k);
// popc of that (restricted to the counted lanes) is the load of bank v, and the congestion is
// the warp maximum (__reduce_max_sync).  Five VOTE + five LOP3 + POPC + REDUX per access.
struct LaneSel {
    uint32_t nsel[5];        // bit k of lane ? 0 : ~0
    __device__ __forceinline__ explicit LaneSel(uint32_t lane) {
#pragma unroll
        for (int k = 0; k < 5; ++k) nsel[k] = ((lane >> k) & 1u) ? 0u : 0xffffffffu;
    }
};

__device__ __forceinline__ uint32_t max_bank_load(uint32_t bank, uint32_t counted, const LaneSel &ls) {
    uint32_t m = counted;
#pragma unroll
    for (int k = 0; k < 5; ++k) m &= __ballot_sync(kFull, (bank >> k) & 1u) ^ ls.nsel[k];
    return __reduce_max_sync(kFull, __popc(m));
}

// Merged requests: lanes of `active` that carry the first occurrence of their
// 10-bit key (the logical cell row*32 + col; every address map is injective on cells).
__device__ __forceinline__ uint32_t first_occurrences(uint32_t key, uint32_t active, uint32_t lane) {
    uint32_t same = active;
#pragma unroll
    for (int k = 0; k < 10; ++k) {
        const uint32_t b = __ballot_sync(kFull, (key >> k) & 1u);
        same &= ((key >> k) & 1u) ? b : ~b;
    }
    const bool leader = (same & ((1u << lane) - 1u)) == 0u;
    return __ballot_sync(kFull, leader) & active;
}

}  // namespace rapk
