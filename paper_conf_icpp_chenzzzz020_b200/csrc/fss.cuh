// fss.cuh -- one-round secure comparison by function secret sharing (SURVEY 8(f) f3,
// DESIGN.md R22).  Distributed comparison function (DCF) of Boyle et al., "Function Secret
// Sharing for Mixed-Mode and Fixed-Point Secure Computation" (EUROCRYPT 2021), Fig. 1, with
// 128-bit seeds and a ChaCha20 block as the length-doubling PRG G, output group Z_2^64.
//
// DReLU(x) from ONE opening: the dealer masks x with a random r (additive shares r_b), the parties
// open xhat = x + r, and with c = MSB(xhat), xhat' = xhat mod 2^63, s = MSB(r):
//     MSB(x) = c ^ s ^ [xhat' < r mod 2^63]
// where [xhat' < alpha] comes from a DCF key with alpha = r mod 2^63 and payload beta = 1 - 2s, so
// the shares sA_b + Eval(b, k_b, xhat') are arithmetic shares of s ^ borrow (no multiplication).
//
// Material per element and party (structure of arrays: word w of element e at mat[w * n + e]):
//   w = 0 r_b, 1 sA_b, 2..3 root seed (lo, hi), then per level i = 1..63: s_CW lo, s_CW hi, V_CW,
//   t_CW^L | t_CW^R << 1; then CW^(64).  FSS_WORDS = 4 * 63 + 5 = 257 words.
// Streams (R11 keys): r = PRG("FR"), r_0 = PRG("F0"), sA_0 = PRG("FS"), root seeds
// PRG64("K0")[2e, 2e+1], PRG64("K1")[2e, 2e+1].
#pragma once
#include "ops.cuh"

namespace psml {

constexpr int FSS_BITS = 63;
constexpr int FSS_WORDS = 4 * FSS_BITS + 5;
constexpr uint32_t TAG_FR = 0x00005246u, TAG_F0 = 0x00003046u, TAG_FS = 0x00005346u, TAG_K0 = 0x0000304Bu,
                   TAG_K1 = 0x0000314Bu, TAG_DCFG = 0x47464344u;

struct S128 {
    uint64_t lo, hi;
};

// G(s) = (s^L, v^L, t^L, s^R, v^R, t^R): ChaCha20 block keyed by the 128-bit seed (|| 16 zero
// bytes), counter 0, nonce "DCFG" || 0.  Words 0-3 s^L, 4-7 s^R, 8-9 v^L, 10-11 v^R, bit 0 of 12 / 13.
__device__ __forceinline__ void dcf_G(const S128 s, S128 &sL, uint64_t &vL, int &tL, S128 &sR, uint64_t &vR, int &tR) {
    const uint32_t k0 = (uint32_t)s.lo, k1 = (uint32_t)(s.lo >> 32), k2 = (uint32_t)s.hi, k3 = (uint32_t)(s.hi >> 32);
    uint32_t x0 = 0x61707865u, x1 = 0x3320646eu, x2 = 0x79622d32u, x3 = 0x6b206574u;
    uint32_t x4 = k0, x5 = k1, x6 = k2, x7 = k3, x8 = 0, x9 = 0, x10 = 0, x11 = 0;
    uint32_t x12 = 0, x13 = TAG_DCFG, x14 = 0, x15 = 0;
#pragma unroll
    for (int r = 0; r < 10; ++r) {
        PSML_QR(x0, x4, x8, x12); PSML_QR(x1, x5, x9, x13);
        PSML_QR(x2, x6, x10, x14); PSML_QR(x3, x7, x11, x15);
        PSML_QR(x0, x5, x10, x15); PSML_QR(x1, x6, x11, x12);
        PSML_QR(x2, x7, x8, x13); PSML_QR(x3, x4, x9, x14);
    }
    x0 += 0x61707865u; x1 += 0x3320646eu; x2 += 0x79622d32u; x3 += 0x6b206574u;
    x4 += k0; x5 += k1; x6 += k2; x7 += k3;
    x13 += TAG_DCFG;
    sL.lo = ((uint64_t)x1 << 32) | x0;
    sL.hi = ((uint64_t)x3 << 32) | x2;
    sR.lo = ((uint64_t)x5 << 32) | x4;
    sR.hi = ((uint64_t)x7 << 32) | x6;
    vL = ((uint64_t)x9 << 32) | x8;
    vR = ((uint64_t)x11 << 32) | x10;
    tL = (int)(x12 & 1);
    tR = (int)(x13 & 1);
}

__device__ __forceinline__ uint64_t neg_if(int t, uint64_t v) { return t ? (uint64_t)0 - v : v; }

// Dealer (offline): Gen of Fig. 1 for every element; both parties' material.
static __global__ void __launch_bounds__(128) fss_dealer_kernel(PrgKey kr, PrgKey kr0, PrgKey ks0, PrgKey kk0, PrgKey kk1,
                                                         int64_t n, int64_t e_lo, int64_t e_hi, int64_t eoff,
                                                         uint64_t *__restrict__ mat0,
                                                         uint64_t *__restrict__ mat1) {
    // elements [e_lo, e_hi) of an n-element material (plane pitch n); element e draws stream
    // element es = e + eoff (eoff != 0: a strong-scaling row-slice of a global stream, R28)
    kr = live_key(kr); kr0 = live_key(kr0); ks0 = live_key(ks0); kk0 = live_key(kk0); kk1 = live_key(kk1);
    for (int64_t e = e_lo + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < e_hi; e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t es = e + eoff;
        const uint64_t r = prg_elem<uint64_t>(kr, es), r0 = prg_elem<uint64_t>(kr0, es), sa0 = prg_elem<uint64_t>(ks0, es);
        S128 s[2];
        s[0].lo = prg_elem<uint64_t>(kk0, 2 * es); s[0].hi = prg_elem<uint64_t>(kk0, 2 * es + 1);
        s[1].lo = prg_elem<uint64_t>(kk1, 2 * es); s[1].hi = prg_elem<uint64_t>(kk1, 2 * es + 1);
        const uint64_t sbit = r >> 63, alpha = r & (((uint64_t)1 << FSS_BITS) - 1);
        const uint64_t beta = (uint64_t)1 - 2 * sbit;
        mat0[e] = r0; mat1[e] = r - r0;
        mat0[n + e] = sa0; mat1[n + e] = sbit - sa0;
        mat0[2 * n + e] = s[0].lo; mat0[3 * n + e] = s[0].hi;
        mat1[2 * n + e] = s[1].lo; mat1[3 * n + e] = s[1].hi;
        int t0 = 0, t1 = 1;
        uint64_t Va = 0;
        for (int i = 1; i <= FSS_BITS; ++i) {
            S128 sL0, sR0, sL1, sR1;
            uint64_t vL0, vR0, vL1, vR1;
            int tL0, tR0, tL1, tR1;
            dcf_G(s[0], sL0, vL0, tL0, sR0, vR0, tR0);
            dcf_G(s[1], sL1, vL1, tL1, sR1, vR1, tR1);
            const int ai = (int)((alpha >> (FSS_BITS - i)) & 1);
            const S128 lose0 = ai ? sL0 : sR0, lose1 = ai ? sL1 : sR1;
            const uint64_t vlose0 = ai ? vL0 : vR0, vlose1 = ai ? vL1 : vR1;
            const uint64_t vkeep0 = ai ? vR0 : vL0, vkeep1 = ai ? vR1 : vL1;
            const S128 scw{lose0.lo ^ lose1.lo, lose0.hi ^ lose1.hi};
            uint64_t Vcw = neg_if(t1, vlose1 - vlose0 - Va);
            if (ai) Vcw += neg_if(t1, beta);
            Va = Va - vkeep1 + vkeep0 + neg_if(t1, Vcw);
            const int tcwL = tL0 ^ tL1 ^ ai ^ 1, tcwR = tR0 ^ tR1 ^ ai;
            const int64_t o = 4 + 4 * (int64_t)(i - 1);
            mat0[o * n + e] = mat1[o * n + e] = scw.lo;
            mat0[(o + 1) * n + e] = mat1[(o + 1) * n + e] = scw.hi;
            mat0[(o + 2) * n + e] = mat1[(o + 2) * n + e] = Vcw;
            mat0[(o + 3) * n + e] = mat1[(o + 3) * n + e] = (uint64_t)(tcwL | (tcwR << 1));
            const int tcwKeep = ai ? tcwR : tcwL;
            S128 k0 = ai ? sR0 : sL0, k1 = ai ? sR1 : sL1;
            if (t0) { k0.lo ^= scw.lo; k0.hi ^= scw.hi; }
            if (t1) { k1.lo ^= scw.lo; k1.hi ^= scw.hi; }
            const int nt0 = (ai ? tR0 : tL0) ^ (t0 & tcwKeep), nt1 = (ai ? tR1 : tL1) ^ (t1 & tcwKeep);
            s[0] = k0; s[1] = k1; t0 = nt0; t1 = nt1;
        }
        const uint64_t last = neg_if(t1, s[1].lo - s[0].lo - Va);
        mat0[(int64_t)(FSS_WORDS - 1) * n + e] = mat1[(int64_t)(FSS_WORDS - 1) * n + e] = last;
    }
}

// Round 1 (the only opening): party b's message xhat_b = x_b + r_b.  only < 0: both parties.
static __global__ void __launch_bounds__(256) fss_mask_kernel(CPair<uint64_t> x, CPair<uint64_t> mat, int64_t n,
                                                       Pair<uint64_t> msg, int only) {
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n; e += (int64_t)gridDim.x * blockDim.x)
#pragma unroll
        for (int p = 0; p < 2; ++p)
            if (only < 0 || only == p) msg.p[p][e] = x.p[p][e] + mat.p[p][e];
}

// Open xhat = msg_0 + msg_1, then Eval(b, k_b, xhat') and the local DReLU combination.  One
// thread per (element, party); xhat_trace (nullable) receives the opened value.
static __global__ void __launch_bounds__(128) fss_eval_kernel(CPair<uint64_t> msg, CPair<uint64_t> mat, int64_t n,
                                                       Pair<uint64_t> drelu, uint64_t *xhat_trace, int only) {
    const int64_t total = only < 0 ? 2 * n : n;
    for (int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; g < total; g += (int64_t)gridDim.x * blockDim.x) {
        const int b = only < 0 ? (int)(g / n) : only;
        const int64_t e = only < 0 ? g % n : g;
        const uint64_t xhat = msg.p[0][e] + msg.p[1][e];
        if (xhat_trace && b == 0) xhat_trace[e] = xhat;
        const uint64_t *k = mat.p[b];
        const uint64_t c = xhat >> 63, x = xhat & (((uint64_t)1 << FSS_BITS) - 1);
        S128 s{k[2 * n + e], k[3 * n + e]};
        int t = b;
        uint64_t V = 0;
        for (int i = 1; i <= FSS_BITS; ++i) {
            const int64_t o = 4 + 4 * (int64_t)(i - 1);
            const S128 scw{k[o * n + e], k[(o + 1) * n + e]};
            const uint64_t Vcw = k[(o + 2) * n + e], tb = k[(o + 3) * n + e];
            S128 sL, sR;
            uint64_t vL, vR;
            int tL, tR;
            dcf_G(s, sL, vL, tL, sR, vR, tR);
            const int xi = (int)((x >> (FSS_BITS - i)) & 1);
            S128 sn = xi ? sR : sL;
            int tn = xi ? tR : tL;
            const uint64_t v = xi ? vR : vL;
            if (t) {
                sn.lo ^= scw.lo; sn.hi ^= scw.hi;
                tn ^= (int)((tb >> xi) & 1);
            }
            V += neg_if(b, v + (t ? Vcw : 0));
            s = sn;
            t = tn;
        }
        V += neg_if(b, s.lo + (t ? k[(int64_t)(FSS_WORDS - 1) * n + e] : 0));
        const uint64_t sx = k[n + e] + V;                      // [s ^ borrow]_b
        const uint64_t one = (uint64_t)(b == 0);
        const uint64_t msb = c ? one - sx : sx;
        drelu.p[b][e] = one - msb;
    }
}

// Eq. 9 through the FSS ReLU (R22): inputs [z + 1/2 ; z - 1/2] (the public constant added by
// party 0), and y = r[0, n) - r[n, 2n), delta = y - Y.  only < 0: both parties.
static __global__ void __launch_bounds__(256) eq9_prep_kernel(CPair<uint64_t> z, int64_t n, uint64_t half,
                                                              Pair<uint64_t> x, int only) {
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n; e += (int64_t)gridDim.x * blockDim.x)
#pragma unroll
        for (int p = 0; p < 2; ++p)
            if (only < 0 || only == p) {
                const uint64_t h = p == 0 ? half : 0;
                x.p[p][e] = z.p[p][e] + h;
                x.p[p][n + e] = z.p[p][e] - h;
            }
}
static __global__ void __launch_bounds__(256) eq9_combine_kernel(CPair<uint64_t> r, int64_t n, Pair<uint64_t> y,
                                                                 CPair<uint64_t> Y, Pair<uint64_t> delta, int only) {
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n; e += (int64_t)gridDim.x * blockDim.x)
#pragma unroll
        for (int p = 0; p < 2; ++p)
            if (only < 0 || only == p) {
                const uint64_t v = r.p[p][e] - r.p[p][n + e];
                y.p[p][e] = v;
                if (delta.p[p]) delta.p[p][e] = v - Y.p[p][e];
            }
}

// Dealer launch with keys whose step field may live in device memory (CUDA graphs).
// elements [e_lo, e_hi) (e_hi < 0: n) of the n-element material, stream elements e + eoff
static inline psml_status fss_dealer_launch(const DealSeeds &S, uint64_t cid, int64_t n, uint64_t *m0, uint64_t *m1,
                                            cudaStream_t s, const uint32_t *step = nullptr, int64_t e_lo = 0,
                                            int64_t e_hi = -1, int64_t eoff = 0) {
    if (e_hi < 0) e_hi = n;
    if (e_hi <= e_lo) return PSML_OK;
    fss_dealer_kernel<<<grid_for(e_hi - e_lo, 128, 148 * 16), 128, 0, s>>>(
        dkey(S, TAG_FR, cid, step), dkey(S, TAG_F0, cid, step), dkey(S, TAG_FS, cid, step),
        dkey(S, TAG_K0, cid, step), dkey(S, TAG_K1, cid, step), n, e_lo, e_hi, eoff, m0, m1);
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

// Both parties' DReLU shares: mask round + (open, evaluate).  ws: 2 n words (messages).
static inline psml_status fss_drelu_launch(CPair<uint64_t> x, int64_t n, CPair<uint64_t> mat, Pair<uint64_t> d,
                                           uint64_t *xhat, uint64_t *ws, cudaStream_t s) {
    Pair<uint64_t> msg{{ws, ws + n}};
    {
        ProfScope prof(PROF_MSB, s, 8.0 * n * 2 * 3);
        fss_mask_kernel<<<ew_grid(n), EW_THREADS, 0, s>>>(x, mat, n, msg, -1);
        PSML_LAUNCH_CHECK();
    }
    ProfScope prof(PROF_MSB, s, 8.0 * n * 2 * (FSS_WORDS + 3));
    fss_eval_kernel<<<grid_for(2 * n, 128, 148 * 16), 128, 0, s>>>(CPair<uint64_t>{{msg.p[0], msg.p[1]}}, mat, n, d,
                                                                  xhat, -1);
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

}  // namespace psml
