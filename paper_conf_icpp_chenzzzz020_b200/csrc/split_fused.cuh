// split_fused.cuh -- the split deployment's secure activation as ONE kernel per party: compute and
// exchange fused over peer memory (psml::PeerWindow of the pair's peer transport).
//
// The activation's rounds (R27 reduced Kogge-Stone MSB: round 0 and log2(l) levels, the
// B2A word, the Beaver Hadamard x . DReLU) are elementwise, so CTA c of party 0 only ever waits for
// CTA c of party 1 (same grid, same element -> CTA map on both sides): every round each thread
// stores its element's masked words straight into the PEER's window (NVLink stores between GPUs),
// the CTA releases a per-CTA flag in the peer's flag words (system scope), acquires the peer's
// flag for the same round, and reads the peer's words from its own window.  No host round trip,
// no separate exchange kernel, no grid-wide barrier; both grids are <= PW_MAX_CTAS CTAs so they are
// co-resident.  Flags are monotonic: (epoch, chunk, round) with the epoch a device counter
// advanced by the last CTA of each call (graph-replay safe).  Bit-identical to the per-round
// kernels + exchanges (same arithmetic, tested against the oracle).
#pragma once
#include "engine.h"

namespace psml {

struct ChainParty {
    int p;                               // this party
    const uint64_t *x, *mat;             // input share (n, or n/2 in Eq. 9 mode), R27 material
    const uint64_t *U, *V, *Z;           // Hadamard triplet of the n elements
    uint64_t *y, *drelu;                 // ReLU: y, drelu (nullable);  Eq. 9: y (n/2)
    const uint64_t *Ysub;                // Eq. 9: delta = y - Ysub (nullable)
    uint64_t *delta;
    int64_t n;                           // elements of the MSB chain (Eq. 9: 2 x the z count)
    int what;                            // 1 ReLU, 2 Eq. 9
    uint64_t half;
    PeerWindow w;
};

__device__ __forceinline__ uint64_t pw_ld_acquire(const uint64_t *p) {
    uint64_t v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void pw_st_release(uint64_t *p, uint64_t v) {
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// one exchange round of this CTA: every thread's stores to the peer's window are visible before the
// flag; the peer's words for the same round are readable after it
__device__ __forceinline__ void pw_round(const PeerWindow &w, uint64_t v) {
    __threadfence_system();
    __syncthreads();
    if (threadIdx.x == 0) {
        pw_st_release(w.peer_flags + PW_FLAG_BASE + (int64_t)blockIdx.x * PW_FLAG_STRIDE, v);
        const uint64_t *mine = w.my_flags + PW_FLAG_BASE + (int64_t)blockIdx.x * PW_FLAG_STRIDE;
        uint64_t t0 = 0;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
        while (pw_ld_acquire(mine) < v) {
            __nanosleep(64);
            uint64_t t;
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
            if (t - t0 > 60ull * 1000000000ull) __trap();   // a peer that never answers
        }
        __threadfence();
    }
    __syncthreads();
}

// The reduced-prefix level j state update for THIS party from the opened words (R27)
__device__ __forceinline__ void pw_level(int p, int l, int j, uint64_t E, uint64_t Fo, const uint64_t gw[3], uint64_t &G,
                                         uint64_t &P) {
    const MsbLevel v = msb_level(l, j);
    uint64_t aG, aP, bG, bP, cG, cP;
    msb_unpack(v, gw[0], aG, aP);
    msb_unpack(v, gw[1], bG, bP);
    msb_unpack(v, gw[2], cG, cP);
    const uint64_t zG = and_z(p, E & v.MG, Fo & v.MG, aG, bG, cG);
    const uint64_t zP = and_z(p, (E << 1) & v.MP, (Fo << 1) & v.MP, aP, bP, cP);
    const int start = j == 1 ? 0 : 1;
    G = compact_bits(G ^ zG, start);
    P = compact_bits(zP, start);
}
__device__ __forceinline__ void pw_level_msgs(int l, int j, const uint64_t gw[3], uint64_t G, uint64_t P, uint64_t &m0,
                                              uint64_t &m1) {
    const MsbLevel v = msb_level(l, j);
    uint64_t aG, aP, bG, bP;
    msb_unpack(v, gw[0], aG, aP);
    msb_unpack(v, gw[1], bG, bP);
    const uint64_t eG = (P ^ aG) & v.MG, fG = ((G << 1) ^ bG) & v.MG;
    const uint64_t eP = (P ^ aP) & v.MP, fP = ((P << 1) ^ bP) & v.MP;
    m0 = eG | (eP >> 1);
    m1 = fG | (fP >> 1);
}

// l = 64.  Thread t of CTA c handles item i = chunk * (grid * 256) + c * 256 + t: one element
// (ReLU) or the element pair (i, i + n/2) of Eq. 9.  Window: 9 rounds x (grid * 256) slots x 4 words.
__global__ void __launch_bounds__(256) msb_chain_party_kernel(const ChainParty A) {
    constexpr int l = 64, L = 6;
    const int p = A.p;
    const int64_t items = A.what == 2 ? A.n / 2 : A.n;
    const int64_t slots = (int64_t)gridDim.x * blockDim.x;
    const int64_t slot = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const uint64_t epoch = *(volatile const uint64_t *)(A.w.my_flags + PW_EPOCH);
    const int64_t nchunks = (items + slots - 1) / slots;
    const int npe = A.what == 2 ? 2 : 1;   // elements per item
    uint64_t *mywin = (uint64_t *)A.w.my_win, *peerwin = (uint64_t *)A.w.peer_win;
    auto put = [&](int r, int k, uint64_t v) { peerwin[((int64_t)r * 4 + k) * slots + slot] = v; };
    auto got = [&](int r, int k) -> uint64_t { return mywin[((int64_t)r * 4 + k) * slots + slot]; };
    const uint64_t M0 = low_bits(l - 1);
    for (int64_t c = 0; c < nchunks; ++c) {
        const int64_t i = c * slots + slot;
        const bool valid = i < items;
        const uint64_t vbase = ((epoch << 20) + (uint64_t)c) << 5;   // + round + 1
        uint64_t x[2] = {0, 0}, gw[2][3][3] = {}, G[2] = {0, 0}, P[2] = {0, 0}, rB[2] = {0, 0}, rA[2] = {0, 0};
        int64_t e[2] = {0, 0};
        for (int q = 0; q < npe; ++q) {
            e[q] = q == 0 ? i : i + A.n / 2;
            if (!valid) continue;
            const uint64_t half = p == 0 ? A.half : 0;
            x[q] = A.what == 2 ? (q == 0 ? A.x[i] + half : A.x[i] - half) : A.x[i];
#pragma unroll
            for (int g = 0; g < 3; ++g)
#pragma unroll
                for (int k = 0; k < 3; ++k) gw[q][g][k] = A.mat[((int64_t)g * 3 + k) * A.n + e[q]];
            rB[q] = A.mat[(int64_t)9 * A.n + e[q]];
            rA[q] = A.mat[(int64_t)10 * A.n + e[q]];
        }
        // round 0: AND 0 on X = (x_0, 0), Y = (0, x_1)
        uint64_t mm[2][2];
        for (int q = 0; q < npe; ++q) {
            mm[q][0] = ((p == 0 ? x[q] : 0) ^ gw[q][0][0]) & M0;
            mm[q][1] = ((p == 1 ? x[q] : 0) ^ gw[q][0][1]) & M0;
            put(0, 2 * q, mm[q][0]);
            put(0, 2 * q + 1, mm[q][1]);
        }
        pw_round(A.w, vbase + 1);
        for (int q = 0; q < npe; ++q) {
            G[q] = and_z(p, mm[q][0] ^ got(0, 2 * q), mm[q][1] ^ got(0, 2 * q + 1), gw[q][0][0], gw[q][0][1], gw[q][0][2]);
            P[q] = x[q];
        }
        // levels 1 .. L: one round each (the packed G and P ANDs)
        for (int j = 1; j <= L; ++j) {
            const int g = j == 1 ? 1 : 2;
            for (int q = 0; q < npe; ++q) {
                pw_level_msgs(l, j, gw[q][g], G[q], P[q], mm[q][0], mm[q][1]);
                put(j, 2 * q, mm[q][0]);
                put(j, 2 * q + 1, mm[q][1]);
            }
            pw_round(A.w, vbase + 1 + j);
            for (int q = 0; q < npe; ++q)
                pw_level(p, l, j, mm[q][0] ^ got(j, 2 * q), mm[q][1] ^ got(j, 2 * q + 1), gw[q][g], G[q], P[q]);
        }
        // B2A: open c = msb ^ rB, [msb]^A = [p = 0] c + (1 - 2c) rA;  DReLU = [p = 0] - [msb]^A
        uint64_t d[2];
        for (int q = 0; q < npe; ++q) {
            const uint64_t bit = ((x[q] >> (l - 1)) & 1) ^ (G[q] & 1);
            mm[q][0] = bit ^ rB[q];
            put(L + 1, q, mm[q][0]);
        }
        pw_round(A.w, vbase + L + 2);
        uint64_t u[2] = {0, 0}, vv[2] = {0, 0}, z[2] = {0, 0};
        for (int q = 0; q < npe; ++q) {
            const uint64_t cc = mm[q][0] ^ got(L + 1, q);
            const uint64_t mA = (p == 0 ? cc : 0) + ((uint64_t)1 - 2 * cc) * rA[q];
            d[q] = (p == 0 ? (uint64_t)1 : 0) - mA;
            if (valid && A.what == 1 && A.drelu) A.drelu[e[q]] = d[q];
            if (valid) { u[q] = A.U[e[q]]; vv[q] = A.V[e[q]]; z[q] = A.Z[e[q]]; }
            mm[q][0] = x[q] - u[q];   // Hadamard x . drelu: E_p, F_p
            mm[q][1] = d[q] - vv[q];
            put(L + 2, 2 * q, mm[q][0]);
            put(L + 2, 2 * q + 1, mm[q][1]);
        }
        pw_round(A.w, vbase + L + 3);
        uint64_t r[2];
        for (int q = 0; q < npe; ++q) {
            const uint64_t E = mm[q][0] + got(L + 2, 2 * q), F = mm[q][1] + got(L + 2, 2 * q + 1);
            r[q] = (uint64_t)p * E * F + E * vv[q] + u[q] * F + z[q];
        }
        if (valid) {
            if (A.what == 1) {
                A.y[i] = r[0];
            } else {
                const uint64_t out = r[0] - r[1];   // ReLU(z + 1/2) - ReLU(z - 1/2)
                A.y[i] = out;
                if (A.delta) A.delta[i] = out - A.Ysub[i];
            }
        }
    }
    // the last CTA out advances the epoch (both parties run the same sequence of calls)
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        const unsigned long long prev = atomicAdd((unsigned long long *)(A.w.my_flags + PW_DONE), 1ull);
        if (prev == gridDim.x - 1) {
            A.w.my_flags[PW_DONE] = 0;
            A.w.my_flags[PW_EPOCH] = epoch + 1;
            __threadfence();
        }
    }
}

// launch: grid = min(PW_MAX_CTAS, items / 256) CTAs on both sides (same n -> same grid)
inline psml_status launch_chain_party(const ChainParty &A, cudaStream_t s) {
    const int64_t items = A.what == 2 ? A.n / 2 : A.n;
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(PW_MAX_CTAS, (items + 255) / 256));
    if ((int64_t)9 * 4 * grid * 256 * 8 > A.w.bytes) return fail(PSML_ERR_STATE, "peer window too small");
    msb_chain_party_kernel<<<grid, 256, 0, s>>>(A);
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

}  // namespace psml
