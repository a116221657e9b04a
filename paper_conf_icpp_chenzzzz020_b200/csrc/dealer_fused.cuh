// dealer_fused.cuh -- the model's whole offline phase for one step in two launches.
//   deal_prg_kernel   one work list over every PRG stream of the step (matrix U/V pairs, Z_0,
//                     Hadamard triplets with Z_1, boolean AND triplets with c_1, daBits); each
//                     thread produces one ChaCha20 block's worth of every stream of its job
//   ring_gemm_cl_grouped<DealerOps> (gemm_cl.cuh) then computes Z_1 = (U_0 + U_1)(V_0 + V_1) - Z_0
//                     for every matrix triplet of the step in one cluster-split-K launch
// Same streams, call ids and arithmetic as the per-item dealer (bit-identical, tested); the step
// field of every call id comes from the model's device word (one captured graph serves all steps).
#pragma once
#include "common.cuh"

#ifndef PSML_DEAL_MINB
#define PSML_DEAL_MINB 5   // min CTAs/SM for the register budget: 5 -> 96 registers, no spills
#endif

namespace psml {

enum { PJ_SINGLE = 0, PJ_PAIR = 1, PJ_HAD = 2, PJ_AND = 3, PJ_DABIT = 4 };

struct PrgJob {
    int kind;
    uint64_t mask;        // PJ_AND: the group's gate bits (reduced prefix, R27)
    uint32_t tag[5];
    uint64_t cid;         // call id with step field 0
    int64_t n;            // elements
    int64_t boff;         // ChaCha20 block offset of element 0 in every stream of the job (the
                          // strong-scaling row-slice of a global stream, R28)
    int64_t blk_begin;    // first global block of this job
    uint64_t *out[6];
};

__device__ __forceinline__ uint64_t cid_with_step(uint64_t cid, const uint32_t *step) {
    return (cid & ~(0xFFFFFFFFull << 24)) | ((uint64_t)(*step) << 24);
}

// 8 consecutive elements e0..e0+7 of one stream (one ChaCha20 block); 16-B vector stores when the
// destination is aligned and the block is whole, else scalar stores up to n.
__device__ __forceinline__ void deal_store8(uint64_t *__restrict__ out, int64_t e0, int64_t n, const uint64_t v[8]) {
    uint64_t *p = out + e0;
    if (e0 + 8 <= n && ((uintptr_t)p & 15) == 0) {
#pragma unroll
        for (int j = 0; j < 8; j += 2) *(ulonglong2 *)(p + j) = make_ulonglong2(v[j], v[j + 1]);
    } else {
#pragma unroll
        for (int j = 0; j < 8; ++j)
            if (e0 + j < n) p[j] = v[j];
    }
}

__device__ __forceinline__ void deal_block(const PrgKey &k, uint32_t b, uint64_t v[8]) {
    uint32_t w[16];
    chacha20_block(k, b, w);
#pragma unroll
    for (int j = 0; j < 8; ++j) v[j] = ((uint64_t)w[2 * j + 1] << 32) | w[2 * j];
}

// Streams 2..4 of a Hadamard (U0 U1 V0 V1 Z0 -> Z1 = (U0+U1)(V0+V1) - Z0) or boolean AND
// (a0 a1 b0 b1 c0 -> c1 = ((a0^a1)&(b0^b1))^c0) job; x holds stream 0, v stream 1.
template <bool HAD>
__device__ __forceinline__ void deal_tail(const PrgJob &J, const DealSeeds &S, uint64_t cid, uint32_t b, int64_t e0, int64_t n,
                                          uint64_t x[8], uint64_t v[8]) {
    uint64_t y[8];
#pragma unroll
    for (int j = 0; j < 8; ++j) x[j] = HAD ? x[j] + v[j] : x[j] ^ v[j];
    deal_block(dkey(S, J.tag[2], cid), b, y);
    deal_store8(J.out[2], e0, n, y);
    deal_block(dkey(S, J.tag[3], cid), b, v);
    deal_store8(J.out[3], e0, n, v);
#pragma unroll
    for (int j = 0; j < 8; ++j) x[j] = HAD ? x[j] * (y[j] + v[j]) : x[j] & (y[j] ^ v[j]);
    deal_block(dkey(S, J.tag[4], cid), b, v);
    deal_store8(J.out[4], e0, n, v);
#pragma unroll
    for (int j = 0; j < 8; ++j) x[j] = HAD ? x[j] - v[j] : x[j] ^ v[j];
    deal_store8(J.out[5], e0, n, x);
}

// Streams of a job are produced one after the other (only the running combination -- U_0 + U_1,
// a_0 ^ a_1, ... -- stays live): 96 registers instead of the 124 that five whole blocks held, so
// the bounded PRG grid (PSML_DEAL_CTAS per SM) leaves part of each SM's register file to the
// online phase it runs beside.
__global__ void __launch_bounds__(128, PSML_DEAL_MINB) deal_prg_kernel(const PrgJob *__restrict__ jobs, int njobs, int64_t blk_first,
                                                           int64_t total_blk, const DealSeeds S, const uint32_t *step) {
    for (int64_t g = blk_first + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; g < total_blk;
         g += (int64_t)gridDim.x * blockDim.x) {
        int lo = 0, hi = njobs - 1;   // last job with blk_begin <= g
        while (lo < hi) {
            const int mid = (lo + hi + 1) >> 1;
            if (jobs[mid].blk_begin <= g) lo = mid; else hi = mid - 1;
        }
        const PrgJob &J = jobs[lo];
        const int64_t b = g - J.blk_begin, e0 = b * 8, n = J.n;
        const uint32_t ctr = (uint32_t)(b + J.boff);   // stream block of local block b
        const uint64_t cid = cid_with_step(J.cid, step);
        const int kind = J.kind;
        uint64_t v[8], x[8], y[8];
        deal_block(dkey(S, J.tag[0], cid), ctr, v);
        if (kind == PJ_DABIT) {
#pragma unroll
            for (int j = 0; j < 8; ++j) { x[j] = v[j] & 1; }
            deal_store8(J.out[0], e0, n, x);
            deal_block(dkey(S, J.tag[1], cid), ctr, v);
#pragma unroll
            for (int j = 0; j < 8; ++j) { v[j] &= 1; x[j] ^= v[j]; }
            deal_store8(J.out[1], e0, n, v);
            deal_block(dkey(S, J.tag[2], cid), ctr, v);   // r^A_0
            deal_store8(J.out[2], e0, n, v);
#pragma unroll
            for (int j = 0; j < 8; ++j) x[j] -= v[j];                    // r^A_1 = (r0 ^ r1) - r^A_0
            deal_store8(J.out[3], e0, n, x);
            continue;
        }
        if (kind == PJ_AND) {   // a0 a1 b0 b1 c0 -> c1 = ((a0^a1)&(b0^b1))^c0, every word masked
            const uint64_t mk = J.mask;
#pragma unroll
            for (int j = 0; j < 8; ++j) { v[j] &= mk; x[j] = v[j]; }
            deal_store8(J.out[0], e0, n, v);
            deal_block(dkey(S, J.tag[1], cid), ctr, v);
#pragma unroll
            for (int j = 0; j < 8; ++j) { v[j] &= mk; x[j] ^= v[j]; }
            deal_store8(J.out[1], e0, n, v);
            deal_block(dkey(S, J.tag[2], cid), ctr, y);
#pragma unroll
            for (int j = 0; j < 8; ++j) y[j] &= mk;
            deal_store8(J.out[2], e0, n, y);
            deal_block(dkey(S, J.tag[3], cid), ctr, v);
#pragma unroll
            for (int j = 0; j < 8; ++j) { v[j] &= mk; x[j] &= y[j] ^ v[j]; }
            deal_store8(J.out[3], e0, n, v);
            deal_block(dkey(S, J.tag[4], cid), ctr, v);
#pragma unroll
            for (int j = 0; j < 8; ++j) { v[j] &= mk; x[j] ^= v[j]; }
            deal_store8(J.out[4], e0, n, v);
            deal_store8(J.out[5], e0, n, x);
            continue;
        }
        deal_store8(J.out[0], e0, n, v);
        if (kind == PJ_SINGLE) continue;
#pragma unroll
        for (int j = 0; j < 8; ++j) x[j] = v[j];
        deal_block(dkey(S, J.tag[1], cid), ctr, v);
        deal_store8(J.out[1], e0, n, v);
        if (kind == PJ_PAIR) continue;
        deal_tail<true>(J, S, cid, ctr, e0, n, x, v);   // PJ_HAD
    }
}

}  // namespace psml
