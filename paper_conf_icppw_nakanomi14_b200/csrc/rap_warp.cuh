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
// __ballot_sync of the bit selected by M.  Written as and + setp + vote so that ptxas turns the
// bit tests of up to 7 ballots of one value into a single R2P (register -> predicates) instead
// of SHF + LOP3 + ISETP per bit (the compiler's lowering of __ballot_sync((x >> k) & 1)).
template <uint32_t M>
__device__ __forceinline__ uint32_t ballot_bit(uint32_t x) {
    uint32_t v;
    asm volatile("{\n\t.reg .pred p;\n\t.reg .b32 t;\n\tand.b32 t, %1, %2;\n\tsetp.ne.u32 p, t, 0;\n\t"
                 "vote.sync.ballot.b32 %0, p, 0xffffffff;\n\t}"
                 : "=r"(v) : "r"(x), "n"(M));
    return v;
}

// B[k] = ballot(bit k of x), k = 0..4 (only bits 0..4 of x are read: x mod 32)
__device__ __forceinline__ void ballot_planes5(uint32_t x, uint32_t (&B)[5]) {
    B[0] = ballot_bit<1u>(x);
    B[1] = ballot_bit<2u>(x);
    B[2] = ballot_bit<4u>(x);
    B[3] = ballot_bit<8u>(x);
    B[4] = ballot_bit<16u>(x);
}

// ballot of ((x & m) == 0): one LOP3 with a predicate output + VOTE
__device__ __forceinline__ uint32_t ballot_zero(uint32_t x, uint32_t m) {
    uint32_t v;
    asm volatile("{\n\t.reg .pred p;\n\t.reg .b32 t;\n\tand.b32 t, %1, %2;\n\tsetp.eq.u32 p, t, 0;\n\t"
                 "vote.sync.ballot.b32 %0, p, 0xffffffff;\n\t}"
                 : "=r"(v) : "r"(x), "r"(m));
    return v;
}

// RAP_FMA_XOR (default 1): x ^ nsel_k, with nsel_k all-zero or all-one per lane, is evaluated as
// the integer multiply-add x * (nsel_k | 1) + nsel_k -- x when nsel_k = 0, -x - 1 = ~x when
// nsel_k = ~0 -- i.e. an IMAD on the FMA pipe; the evaluators are bound by the ALU pipe (LOP3),
// and the remaining ANDs then take three operands per LOP3.
#ifndef RAP_FMA_XOR
#define RAP_FMA_XOR 1
#endif

struct LaneSel {
    uint32_t nsel[5];        // bit k of lane ? 0 : ~0
    uint32_t flip[5];        // nsel | 1: +1 or -1
    __device__ __forceinline__ explicit LaneSel(uint32_t lane) {
#pragma unroll
        for (int k = 0; k < 5; ++k) {
            nsel[k] = ((lane >> k) & 1u) ? 0u : 0xffffffffu;
            flip[k] = nsel[k] | 1u;
        }
    }
    // x ^ nsel[k]
    __device__ __forceinline__ uint32_t sel(uint32_t x, int k) const {
#if RAP_FMA_XOR
        return x * flip[k] + nsel[k];
#else
        return x ^ nsel[k];
#endif
    }
};

// counted AND_k (B_k ^ nsel_k): lanes whose bank (bit planes B) equals this lane's index
__device__ __forceinline__ uint32_t lanes_equal(const uint32_t (&B)[5], uint32_t counted, const LaneSel &ls) {
#if RAP_FMA_XOR
    const uint32_t t0 = ls.sel(B[0], 0), t1 = ls.sel(B[1], 1), t2 = ls.sel(B[2], 2), t3 = ls.sel(B[3], 3),
                   t4 = ls.sel(B[4], 4);
    return ((counted & t0 & t1) & t2 & t3) & t4;
#else
    uint32_t m = counted;
#pragma unroll
    for (int k = 0; k < 5; ++k) m &= B[k] ^ ls.nsel[k];
    return m;
#endif
}

__device__ __forceinline__ uint32_t max_bank_load(uint32_t bank, uint32_t counted, const LaneSel &ls) {
    uint32_t B[5];
    ballot_planes5(bank, B);
    return __reduce_max_sync(kFull, __popc(lanes_equal(B, counted, ls)));
}

// Merged requests: lanes of `active` that carry the first occurrence of their
// 10-bit key (the logical cell row*32 + col; every address map is injective on cells).
__device__ __forceinline__ uint32_t first_occurrences(uint32_t key, uint32_t active, uint32_t lane) {
    uint32_t b[5];
    ballot_planes5(key & 31u, b);
    uint32_t same = active;
#pragma unroll
    for (int k = 0; k < 5; ++k) same &= ((key >> k) & 1u) ? b[k] : ~b[k];
    ballot_planes5(key >> 5, b);
#pragma unroll
    for (int k = 0; k < 5; ++k) same &= ((key >> (k + 5)) & 1u) ? b[k] : ~b[k];
    return ballot_zero(same, (1u << lane) - 1u) & active;
}

}  // namespace rapk
