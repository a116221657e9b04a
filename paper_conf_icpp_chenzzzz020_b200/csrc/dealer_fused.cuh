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

namespace psml {

enum { PJ_SINGLE = 0, PJ_PAIR = 1, PJ_HAD = 2, PJ_AND = 3, PJ_DABIT = 4 };

struct PrgJob {
    int kind;
    uint32_t tag[5];
    uint64_t cid;         // call id with step field 0
    int64_t n;            // elements
    int64_t blk_begin;    // first global block of this job
    uint64_t *out[6];
};

__device__ __forceinline__ uint64_t cid_with_step(uint64_t cid, const uint32_t *step) {
    return (cid & ~(0xFFFFFFFFull << 24)) | ((uint64_t)(*step) << 24);
}

__global__ void __launch_bounds__(128) deal_prg_kernel(const PrgJob *__restrict__ jobs, int njobs, int64_t total_blk,
                                                        uint64_t seed, const uint32_t *step) {
    for (int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; g < total_blk;
         g += (int64_t)gridDim.x * blockDim.x) {
        int lo = 0, hi = njobs - 1;   // last job with blk_begin <= g
        while (lo < hi) {
            const int mid = (lo + hi + 1) >> 1;
            if (jobs[mid].blk_begin <= g) lo = mid; else hi = mid - 1;
        }
        const PrgJob &J = jobs[lo];
        const int64_t b = g - J.blk_begin;
        const uint64_t cid = cid_with_step(J.cid, step);
        const int ns = J.kind == PJ_SINGLE ? 1 : J.kind == PJ_PAIR ? 2 : J.kind == PJ_DABIT ? 3 : 5;
        uint32_t w[5][16];
#pragma unroll
        for (int i = 0; i < 5; ++i)
            if (i < ns) chacha20_block(make_key(seed, J.tag[i], cid), (uint32_t)b, w[i]);
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            const int64_t e = b * 8 + j;
            if (e >= J.n) break;
            uint64_t v[5];
#pragma unroll
            for (int i = 0; i < 5; ++i) v[i] = i < ns ? (((uint64_t)w[i][2 * j + 1] << 32) | w[i][2 * j]) : 0;
            switch (J.kind) {
            case PJ_SINGLE: J.out[0][e] = v[0]; break;
            case PJ_PAIR: J.out[0][e] = v[0]; J.out[1][e] = v[1]; break;
            case PJ_HAD:   // U0 U1 V0 V1 Z0 -> Z1
                J.out[0][e] = v[0]; J.out[1][e] = v[1]; J.out[2][e] = v[2]; J.out[3][e] = v[3];
                J.out[4][e] = v[4]; J.out[5][e] = (v[0] + v[1]) * (v[2] + v[3]) - v[4];
                break;
            case PJ_AND:   // a0 a1 b0 b1 c0 -> c1
                J.out[0][e] = v[0]; J.out[1][e] = v[1]; J.out[2][e] = v[2]; J.out[3][e] = v[3];
                J.out[4][e] = v[4]; J.out[5][e] = ((v[0] ^ v[1]) & (v[2] ^ v[3])) ^ v[4];
                break;
            default: {     // daBit: R0 R1 RA -> rB0, rB1, rA0, rA1
                const uint64_t r0 = v[0] & 1, r1 = v[1] & 1;
                J.out[0][e] = r0; J.out[1][e] = r1; J.out[2][e] = v[2]; J.out[3][e] = (r0 ^ r1) - v[2];
            }
            }
        }
    }
}

}  // namespace psml
