// gemm_simt.cuh -- CUDA-core ring GEMM in Z_{2^l} (l = 64: uint64 IMAD.WIDE chains; l = 32:
// uint32 IMAD) with pluggable operand loaders and epilogues.
//
// The loaders fuse the Beaver opening and the Eq. 8 K-concatenation of PAPER.md L175:
//   party i computes C_i = [i.E + U_i | E] . [F ; V_i] + Z_i with E = E_0 + E_1, F = F_0 + F_1
// read straight from both parties' masked messages, so D' = i.E + U_i is never materialised.
// Two kernels:
//   ring_gemm_tiled  BM x BN tiles, register-blocked TM x TN per thread, double-buffered smem
//   ring_gemv        one warp per output row for N <= 16 (w^T x shapes of BASELINE configs 1-2,
//                    the MLP output layer, the CNN conv im2col GEMM with N = C_out = 16)
// Both support split-K with exact uint64/uint32 atomics (ring addition is associative and
// exact), finished by ring_gemm_finalize which applies the epilogue.
#pragma once
#include <algorithm>
#include <cstdlib>

#include "common.cuh"

namespace psml {

// ring multiply-accumulate with split accumulators for u64
template <typename T> struct RingAcc {
    T v;
    __device__ __forceinline__ void zero() { v = 0; }
    __device__ __forceinline__ void mac(T a, T b) { v += a * b; }
    __device__ __forceinline__ T value() const { return v; }
};
template <> struct RingAcc<uint64_t> {
    uint64_t w;        // sum of lo.lo (64-bit, IMAD.WIDE.U32 with accumulate)
    uint32_t x1, x2;   // sums of lo.hi and hi.lo (mod 2^32), two chains
    __device__ __forceinline__ void zero() { w = 0; x1 = 0; x2 = 0; }
    __device__ __forceinline__ void mac(uint64_t a, uint64_t b) {
        const uint32_t al = (uint32_t)a, ah = (uint32_t)(a >> 32), bl = (uint32_t)b, bh = (uint32_t)(b >> 32);
        asm("mad.wide.u32 %0, %1, %2, %0;" : "+l"(w) : "r"(al), "r"(bl));
        asm("mad.lo.u32 %0, %1, %2, %0;" : "+r"(x1) : "r"(al), "r"(bh));
        asm("mad.lo.u32 %0, %1, %2, %0;" : "+r"(x2) : "r"(ah), "r"(bl));
    }
    __device__ __forceinline__ uint64_t value() const { return w + ((uint64_t)(x1 + x2) << 32); }
};

// ---------------------------------------------------------------------------------------------
// operand/epilogue policies.  Each provides:
//   nparty, M, N, Kext; T a(p, m, k); T b(p, k, n); void store(p, m, n, T acc)
// ---------------------------------------------------------------------------------------------
template <typename T>
struct PlainOps {
    const T *A, *B;
    T *C;
    int64_t M, N, Kext;
    static constexpr int nparty = 1;
    __device__ __forceinline__ T a(int, int64_t m, int64_t k) const { return A[m * Kext + k]; }
    __device__ __forceinline__ T b(int, int64_t k, int64_t n) const { return B[k * N + n]; }
    __device__ __forceinline__ T zload(int, int64_t, int64_t) const { return 0; }
    __device__ __forceinline__ void put(int, int64_t m, int64_t n, T acc, T) const { C[m * N + n] = acc; }
    __device__ __forceinline__ void store(int, int64_t m, int64_t n, T acc) const { C[m * N + n] = acc; }
};

// Dealer: Z = (U_0 + U_1)(V_0 + V_1); Z_1 = Z - Z_0 with Z_0 = PRG("Z0") already written by the
// vectorised PRG kernel (Eqs. 2-3, R4).
template <typename T>
struct DealerOps {
    const T *U0, *U1, *V0, *V1;
    const T *Z0;
    T *Z1;
    int64_t M, N, Kext;
    static constexpr int nparty = 1;
    __device__ __forceinline__ T a(int, int64_t m, int64_t k) const {
        return U0[m * Kext + k] + U1[m * Kext + k];
    }
    __device__ __forceinline__ T b(int, int64_t k, int64_t n) const {
        return V0[k * N + n] + V1[k * N + n];
    }
    __device__ __forceinline__ T zload(int, int64_t m, int64_t n) const { return Z0[m * N + n]; }
    __device__ __forceinline__ void put(int, int64_t m, int64_t n, T acc, T z) const { Z1[m * N + n] = acc - z; }
    __device__ __forceinline__ void store(int, int64_t m, int64_t n, T acc) const {
        Z1[m * N + n] = acc - Z0[m * N + n];
    }
};

// Beaver product, both parties, Eq. 8 shape.  E/F are opened on the fly from the two parties'
// messages mE[0], mE[1] (M x K) and mF[0], mF[1] (K x N).  form 0 (BJ canonical):
//   [i.E + U_i | E] . [F ; V_i];  form 1 (Eq. 6/8): [A_i - i.E | E] . [F ; B_i].
template <typename T, int FORM = 0>
struct BeaverOps {
    const T *mE0, *mE1, *mF0, *mF1;
    const T *U[2], *V[2], *Z[2];
    const T *A[2], *B[2];   // only for form 1 (op(A) / op(B) layouts, see transA/transB)
    T *C[2];
    int64_t M, N, K, Kext;  // Kext = 2K
    int transA, transB, trunc;
    static constexpr int form = FORM;   // compile time: no branch in the loaders
    static constexpr int nparty = 2;
    // Branch-free loaders (every load issued unconditionally at a valid address, the result
    // selected afterwards) so a thread's operand loads overlap instead of serialising.
    __device__ __forceinline__ T a(int p, int64_t m, int64_t k) const {
        const bool first = k < K;
        const int64_t kk = first ? k : k - K, i = m * K + kk;
        const T e = mE0[i] + mE1[i];
        const T x = form == 0 ? U[p][i] : A[p][transA ? kk * M + m : i];
        return first ? (form == 0 ? (T)((T)p * e + x) : (T)(x - (T)p * e)) : e;
    }
    __device__ __forceinline__ T b(int p, int64_t k, int64_t n) const {
        const bool first = k < K;
        const int64_t kk = first ? k : k - K, i = kk * N + n;
        const T *second = form == 0 ? V[p] + i : B[p] + (transB ? n * K + kk : i);
        const T x = *(first ? mF0 + i : second), y = mF1[i];
        return first ? (T)(x + y) : x;
    }
    __device__ __forceinline__ T zload(int p, int64_t m, int64_t n) const { return Z[p][m * N + n]; }
    __device__ __forceinline__ void put(int p, int64_t m, int64_t n, T acc, T z) const {
        C[p][m * N + n] = trunc_share<T>(acc + z, p, trunc);
    }
    __device__ __forceinline__ void store(int p, int64_t m, int64_t n, T acc) const {
        T c = acc + Z[p][m * N + n];
        C[p][m * N + n] = trunc_share<T>(c, p, trunc);
    }
};

// Co-resident Beaver product with the mask round fused into the operand loads: the opened
// E = (op(A)_0 - U_0) + (op(A)_1 - U_1) and F likewise are formed where the GEMM reads them (the
// same ring arithmetic as mask kernel + open; no message buffers, one launch less per product).
// a_kmajor()/b_kmajor() tell the loaders which index is contiguous so transposed operands stay
// coalesced.
template <typename T>
struct BeaverFusedOps {
    const T *A[2], *B[2], *U[2], *V[2], *Z[2];
    T *C[2];
    int64_t M, N, K, Kext;
    int transA, transB, trunc;
    static constexpr int nparty = 2;
    __device__ __forceinline__ bool a_kmajor() const { return !transA; }
    __device__ __forceinline__ bool b_nmajor() const { return !transB; }
    __device__ __forceinline__ T opA(int p, int64_t m, int64_t k) const {
        return transA ? A[p][k * M + m] : A[p][m * K + k];
    }
    __device__ __forceinline__ T opB(int p, int64_t k, int64_t n) const {
        return transB ? B[p][n * K + k] : B[p][k * N + n];
    }
    __device__ __forceinline__ T a(int p, int64_t m, int64_t k) const {
        const bool first = k < K;
        const int64_t kk = first ? k : k - K, u = m * K + kk;
        const T u0 = U[0][u], u1 = U[1][u];
        const T e = (opA(0, m, kk) - u0) + (opA(1, m, kk) - u1);
        return first ? (T)((T)p * e + (p ? u1 : u0)) : e;
    }
    __device__ __forceinline__ T b(int p, int64_t k, int64_t n) const {
        const bool first = k < K;
        const int64_t kk = first ? k : k - K, i = kk * N + n;
        const T v0 = V[0][i], v1 = V[1][i];
        const T f = (opB(0, kk, n) - v0) + (opB(1, kk, n) - v1);
        return first ? f : (p ? v1 : v0);
    }
    __device__ __forceinline__ T zload(int p, int64_t m, int64_t n) const { return Z[p][m * N + n]; }
    __device__ __forceinline__ void put(int p, int64_t m, int64_t n, T acc, T z) const {
        C[p][m * N + n] = trunc_share<T>(acc + z, p, trunc);
    }
    __device__ __forceinline__ void store(int p, int64_t m, int64_t n, T acc) const {
        C[p][m * N + n] = trunc_share<T>(acc + Z[p][m * N + n], p, trunc);
    }
};

template <class Ops> __device__ __forceinline__ bool ops_a_kmajor(const Ops &o, int) { return true; }
template <class Ops> __device__ __forceinline__ bool ops_b_nmajor(const Ops &o, int) { return true; }
template <typename T> __device__ __forceinline__ bool ops_a_kmajor(const BeaverFusedOps<T> &o, int) { return o.a_kmajor(); }
template <typename T> __device__ __forceinline__ bool ops_b_nmajor(const BeaverFusedOps<T> &o, int) { return o.b_nmajor(); }

// One party of the split deployment: own messages (mE0/mF0 = sent) + the peer's (mE1/mF1 =
// received); same arithmetic as BeaverOps for party `party`.
template <typename T>
struct BeaverOps1 {
    const T *mE0, *mE1, *mF0, *mF1;
    const T *U, *V, *Z;
    T *C;
    int64_t M, N, K, Kext;
    int party, trunc;
    static constexpr int nparty = 1;
    __device__ __forceinline__ T a(int, int64_t m, int64_t k) const {
        const bool first = k < K;
        const int64_t kk = first ? k : k - K, i = m * K + kk;
        const T e = mE0[i] + mE1[i], u = U[i];
        return first ? (T)((T)party * e + u) : e;
    }
    __device__ __forceinline__ T b(int, int64_t k, int64_t n) const {
        const bool first = k < K;
        const int64_t kk = first ? k : k - K, i = kk * N + n;
        const T x = *(first ? mF0 + i : V + i), y = mF1[i];
        return first ? (T)(x + y) : x;
    }
    __device__ __forceinline__ T zload(int, int64_t m, int64_t n) const { return Z[m * N + n]; }
    __device__ __forceinline__ void put(int, int64_t m, int64_t n, T acc, T z) const {
        C[m * N + n] = trunc_share<T>(acc + z, party, trunc);
    }
    __device__ __forceinline__ void store(int, int64_t m, int64_t n, T acc) const {
        C[m * N + n] = trunc_share<T>(acc + Z[m * N + n], party, trunc);
    }
};

// Convolution as im2col ring GEMM with the mask applied to the UN-EXPANDED input (R17):
// E_X = E_0 + E_1 over B x (C H W); im2col row r = (b, oy, ox), col c = (ch, ky, kx).
// transposed = 0: A' = im2col(.)            (rows B*OH*OW, K = C*k*k)   -- conv forward
// transposed = 1: A' = im2col(.)^T          (rows C*k*k,  K = B*OH*OW)  -- weight gradient
struct ConvGeom {
    int C, H, W, k, OH, OW;
    const int32_t *coloff;   // device table: offset of im2col column c = (ch, ky, kx) in a sample
};

// im2col source index of (row r = (b, oy, ox), column c): 32-bit row decomposition (indices of
// the paper's workloads fit in 31 bits) + the precomputed column offset -- no 64-bit divisions.
__device__ __forceinline__ int64_t conv_src(const ConvGeom &g, int64_t r, int64_t c) {
    const uint32_t r32 = (uint32_t)r, plane = (uint32_t)(g.OH * g.OW);
    const uint32_t b = r32 / plane, rem = r32 - b * plane;
    const uint32_t oy = rem / (uint32_t)g.OW, ox = rem - oy * (uint32_t)g.OW;
    return (int64_t)b * ((int64_t)g.C * g.H * g.W) + (int64_t)(oy * (uint32_t)g.W + ox) + g.coloff[c];
}

template <typename T>
struct ConvBeaverOps {
    const T *mE0, *mE1;     // masked raw input messages, B x CHW
    const T *UX[2];         // raw-input masks per party, B x CHW
    const T *mF0, *mF1;     // masked B-operand messages, K x N
    const T *V[2], *Z[2];
    T *C[2];
    ConvGeom g;
    int64_t M, N, K, Kext;
    int transposed, trunc;
    static constexpr int nparty = 2;
    __device__ __forceinline__ int64_t src(int64_t r, int64_t c) const { return conv_src(g, r, c); }
    __device__ __forceinline__ T a(int p, int64_t m, int64_t k) const {
        const bool first = k < K;
        const int64_t kk = first ? k : k - K;
        const int64_t s = transposed ? src(kk, m) : src(m, kk);
        const T e = mE0[s] + mE1[s], u = UX[p][s];
        return first ? (T)((T)p * e + u) : e;
    }
    __device__ __forceinline__ T b(int p, int64_t k, int64_t n) const {
        const bool first = k < K;
        const int64_t kk = first ? k : k - K, i = kk * N + n;
        const T x = *(first ? mF0 + i : V[p] + i), y = mF1[i];
        return first ? (T)(x + y) : x;
    }
    __device__ __forceinline__ T zload(int p, int64_t m, int64_t n) const { return Z[p][m * N + n]; }
    __device__ __forceinline__ void put(int p, int64_t m, int64_t n, T acc, T z) const {
        C[p][m * N + n] = trunc_share<T>(acc + z, p, trunc);
    }
    __device__ __forceinline__ void store(int p, int64_t m, int64_t n, T acc) const {
        T c = acc + Z[p][m * N + n];
        C[p][m * N + n] = trunc_share<T>(c, p, trunc);
    }
};

// Split deployment, one party: E = mE0 + mE1 (this party's message + the peer's), F likewise;
// C = im2col([party.E + U_X | E]) (.^T) . [F ; V] + Z, truncated (same arithmetic as above).
template <typename T>
struct ConvBeaverOps1 {
    const T *mE0, *mE1, *UX, *mF0, *mF1, *V, *Z;
    T *C;
    ConvGeom g;
    int64_t M, N, K, Kext;
    int transposed, trunc, party;
    static constexpr int nparty = 1;
    __device__ __forceinline__ int64_t src(int64_t r, int64_t c) const { return conv_src(g, r, c); }
    __device__ __forceinline__ T a(int, int64_t m, int64_t k) const {
        const bool first = k < K;
        const int64_t kk = first ? k : k - K;
        const int64_t s = transposed ? src(kk, m) : src(m, kk);
        const T e = mE0[s] + mE1[s], u = UX[s];
        return first ? (T)((T)party * e + u) : e;
    }
    __device__ __forceinline__ T b(int, int64_t k, int64_t n) const {
        const bool first = k < K;
        const int64_t kk = first ? k : k - K, i = kk * N + n;
        const T x = *(first ? mF0 + i : V + i), y = mF1[i];
        return first ? (T)(x + y) : x;
    }
    __device__ __forceinline__ T zload(int, int64_t m, int64_t n) const { return Z[m * N + n]; }
    __device__ __forceinline__ void put(int, int64_t m, int64_t n, T acc, T z) const {
        C[m * N + n] = trunc_share<T>(acc + z, party, trunc);
    }
    __device__ __forceinline__ void store(int, int64_t m, int64_t n, T acc) const {
        C[m * N + n] = trunc_share<T>(acc + Z[m * N + n], party, trunc);
    }
};

// Dealer for the conv triplet: Z = im2col(U_0+U_1) (.^T) . (V_0+V_1), Z_1 = Z - PRG("Z0").
template <typename T>
struct ConvDealerOps {
    const T *U0, *U1, *V0, *V1;
    const T *Z0;
    T *Z1;
    ConvGeom g;
    int64_t M, N, Kext;
    int transposed;
    static constexpr int nparty = 1;
    __device__ __forceinline__ int64_t src(int64_t r, int64_t c) const { return conv_src(g, r, c); }
    __device__ __forceinline__ T a(int, int64_t m, int64_t k) const {
        int64_t s = transposed ? src(k, m) : src(m, k);
        return U0[s] + U1[s];
    }
    __device__ __forceinline__ T b(int, int64_t k, int64_t n) const {
        return V0[k * N + n] + V1[k * N + n];
    }
    __device__ __forceinline__ T zload(int, int64_t m, int64_t n) const { return Z0[m * N + n]; }
    __device__ __forceinline__ void put(int, int64_t m, int64_t n, T acc, T z) const { Z1[m * N + n] = acc - z; }
    __device__ __forceinline__ void store(int, int64_t m, int64_t n, T acc) const {
        Z1[m * N + n] = acc - Z0[m * N + n];
    }
};

// ---------------------------------------------------------------------------------------------
// tiled kernel
// ---------------------------------------------------------------------------------------------
template <typename T, int BM, int BN, int BK, int TM, int TN, class Ops>
__global__ void __launch_bounds__((BM / TM) * (BN / TN))
ring_gemm_tiled(Ops ops, int64_t k_per_split, T *__restrict__ partial) {
    constexpr int NT = (BM / TM) * (BN / TN);
    constexpr int A_PER = (BM * BK) / NT;
    constexpr int B_PER = (BK * BN) / NT;
    static_assert(A_PER * NT == BM * BK && B_PER * NT == BK * BN, "tile/thread mismatch");
    __shared__ T As[2][BK][BM];
    __shared__ T Bs[2][BK][BN];

    const int p = blockIdx.z % Ops::nparty;
    const int split = blockIdx.z / Ops::nparty;
    const int64_t m0 = (int64_t)blockIdx.y * BM, n0 = (int64_t)blockIdx.x * BN;
    const int64_t kbeg = (int64_t)split * k_per_split;
    const int64_t kend = min(ops.Kext, kbeg + k_per_split);
    const int tid = threadIdx.x;
    const int tx = tid % (BN / TN), ty = tid / (BN / TN);

    T acc[TM][TN];
#pragma unroll
    for (int i = 0; i < TM; ++i)
#pragma unroll
        for (int j = 0; j < TN; ++j) acc[i][j] = 0;

    T ra[A_PER], rb[B_PER];
    auto load = [&](int64_t k0) {
#pragma unroll
        for (int t = 0; t < A_PER; ++t) {
            int idx = tid + t * NT;
            int mm = idx / BK, kk = idx % BK;          // coalesced along k
            int64_t m = m0 + mm, k = k0 + kk;
            const T v = ops.a(p, m < ops.M ? m : ops.M - 1, k < kend ? k : kend - 1);
            ra[t] = (m < ops.M && k < kend) ? v : (T)0;
        }
#pragma unroll
        for (int t = 0; t < B_PER; ++t) {
            int idx = tid + t * NT;
            int kk = idx / BN, nn = idx % BN;          // coalesced along n
            int64_t k = k0 + kk, n = n0 + nn;
            const T v = ops.b(p, k < kend ? k : kend - 1, n < ops.N ? n : ops.N - 1);
            rb[t] = (n < ops.N && k < kend) ? v : (T)0;
        }
    };
    auto stash = [&](int buf) {
#pragma unroll
        for (int t = 0; t < A_PER; ++t) {
            int idx = tid + t * NT;
            As[buf][idx % BK][idx / BK] = ra[t];
        }
#pragma unroll
        for (int t = 0; t < B_PER; ++t) {
            int idx = tid + t * NT;
            Bs[buf][idx / BN][idx % BN] = rb[t];
        }
    };

    int buf = 0;
    if (kbeg < kend) {
        load(kbeg);
        stash(0);
    }
    __syncthreads();
    for (int64_t k0 = kbeg; k0 < kend; k0 += BK) {
        const bool more = k0 + BK < kend;
        if (more) load(k0 + BK);
#pragma unroll
        for (int kk = 0; kk < BK; ++kk) {
            T av[TM], bv[TN];
#pragma unroll
            for (int i = 0; i < TM; ++i) av[i] = As[buf][kk][ty + i * (BM / TM)];
#pragma unroll
            for (int j = 0; j < TN; ++j) bv[j] = Bs[buf][kk][tx + j * (BN / TN)];
#pragma unroll
            for (int i = 0; i < TM; ++i)
#pragma unroll
                for (int j = 0; j < TN; ++j) acc[i][j] += av[i] * bv[j];
        }
        if (more) {
            stash(buf ^ 1);
            __syncthreads();
            buf ^= 1;
        }
    }
    if (partial == nullptr) {
        // epilogue operands first (clamped, unconditional), then the stores: no serialised loads
        T z[TM][TN];
#pragma unroll
        for (int i = 0; i < TM; ++i)
#pragma unroll
            for (int j = 0; j < TN; ++j) {
                const int64_t m = m0 + ty + i * (BM / TM), n = n0 + tx + j * (BN / TN);
                z[i][j] = ops.zload(p, m < ops.M ? m : ops.M - 1, n < ops.N ? n : ops.N - 1);
            }
#pragma unroll
        for (int i = 0; i < TM; ++i) {
            int64_t m = m0 + ty + i * (BM / TM);
            if (m >= ops.M) continue;
#pragma unroll
            for (int j = 0; j < TN; ++j) {
                int64_t n = n0 + tx + j * (BN / TN);
                if (n < ops.N) ops.put(p, m, n, acc[i][j], z[i][j]);
            }
        }
    } else {
#pragma unroll
        for (int i = 0; i < TM; ++i) {
            int64_t m = m0 + ty + i * (BM / TM);
            if (m >= ops.M) continue;
#pragma unroll
            for (int j = 0; j < TN; ++j) {
                int64_t n = n0 + tx + j * (BN / TN);
                if (n >= ops.N) continue;
                T *dst = partial + ((int64_t)p * ops.M + m) * ops.N + n;
                if (sizeof(T) == 8) atomicAdd((unsigned long long *)dst, (unsigned long long)acc[i][j]);
                else atomicAdd((unsigned int *)dst, (unsigned int)acc[i][j]);
            }
        }
    }
}

// ---------------------------------------------------------------------------------------------
// small-output kernel: 16 x 16 output tile per 256-thread CTA (one output per thread), K in
// chunks of 64 staged in smem with the next chunk prefetched into registers.  For the MLP's
// 128 x 128 products this gives 64-128 CTAs without split-K, i.e. ~K'/64 memory round trips
// instead of the 64 x 64 tile's K'/16 at ~2 warps per SM.
// ---------------------------------------------------------------------------------------------
template <typename T, class Ops>
__global__ void __launch_bounds__(256) ring_gemm_small(Ops ops, int64_t k_per_split, T *__restrict__ partial) {
    constexpr int BM = 16, BN = 16, BK = 64;
    __shared__ T As[2][BM][BK + 1];
    __shared__ T Bs[2][BK][BN];
    const int p = blockIdx.z % Ops::nparty;
    const int split = blockIdx.z / Ops::nparty;
    const int64_t m0 = (int64_t)blockIdx.y * BM, n0 = (int64_t)blockIdx.x * BN;
    const int64_t kbeg = (int64_t)split * k_per_split;
    const int64_t kend = min(ops.Kext, kbeg + k_per_split);
    const int tid = threadIdx.x;
    const int tx = tid & 15, ty = tid >> 4;
    T ra[4], rb[4];
    // thread -> element maps: A 16 x 64 consecutive along k (row-major A) or along m (A^T);
    // B 64 x 16 consecutive along n (row-major B) or along k (B^T)
    const bool ak = ops_a_kmajor(ops, 0), bn = ops_b_nmajor(ops, 0);
    auto amap = [&](int idx, int &mm, int &kk) {
        if (ak) { mm = idx >> 6; kk = idx & 63; } else { mm = idx & 15; kk = idx >> 4; }
    };
    auto bmap = [&](int idx, int &kb, int &nn) {
        if (bn) { kb = idx >> 4; nn = idx & 15; } else { kb = idx & 63; nn = idx >> 6; }
    };
    auto load = [&](int64_t k0) {
#pragma unroll
        for (int t = 0; t < 4; ++t) {
            const int idx = tid + t * 256;
            int mm, kk, kb, nn;
            amap(idx, mm, kk);
            const int64_t m = m0 + mm, k = k0 + kk;
            const T va = ops.a(p, m < ops.M ? m : ops.M - 1, k < kend ? k : kend - 1);
            ra[t] = (m < ops.M && k < kend) ? va : (T)0;
            bmap(idx, kb, nn);
            const int64_t k2 = k0 + kb, n = n0 + nn;
            const T vb = ops.b(p, k2 < kend ? k2 : kend - 1, n < ops.N ? n : ops.N - 1);
            rb[t] = (n < ops.N && k2 < kend) ? vb : (T)0;
        }
    };
    auto stash = [&](int buf) {
#pragma unroll
        for (int t = 0; t < 4; ++t) {
            const int idx = tid + t * 256;
            int mm, kk, kb, nn;
            amap(idx, mm, kk);
            bmap(idx, kb, nn);
            As[buf][mm][kk] = ra[t];
            Bs[buf][kb][nn] = rb[t];
        }
    };
    T acc = 0;
    int buf = 0;
    if (kbeg < kend) { load(kbeg); stash(0); }
    __syncthreads();
    for (int64_t k0 = kbeg; k0 < kend; k0 += BK) {
        const bool more = k0 + BK < kend;
        if (more) load(k0 + BK);
#pragma unroll 16
        for (int kk = 0; kk < BK; ++kk) acc += As[buf][ty][kk] * Bs[buf][kk][tx];
        if (more) {
            stash(buf ^ 1);
            __syncthreads();
            buf ^= 1;
        }
    }
    const int64_t m = m0 + ty, n = n0 + tx;
    if (m < ops.M && n < ops.N) {
        if (partial == nullptr) ops.store(p, m, n, acc);
        else {
            T *dst = partial + ((int64_t)p * ops.M + m) * ops.N + n;
            if (sizeof(T) == 8) atomicAdd((unsigned long long *)dst, (unsigned long long)acc);
            else atomicAdd((unsigned int *)dst, (unsigned int)acc);
        }
    }
}

// ---------------------------------------------------------------------------------------------
// warp-per-row kernel for N <= NN (NN in {1, 2, 4, 8, 16})
// ---------------------------------------------------------------------------------------------
template <typename T>
__device__ __forceinline__ T warp_sum(T v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

template <typename T, int NN, class Ops>
__global__ void __launch_bounds__(256) ring_gemv(Ops ops, int64_t k_per_split, int splits,
                                                 T *__restrict__ partial) {
    const int lane = threadIdx.x & 31;
    const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t rows = ops.M * Ops::nparty * splits;
    if (gw >= rows) return;
    const int split = (int)(gw % splits);
    const int64_t pm = gw / splits;
    const int p = (int)(pm % Ops::nparty);
    const int64_t m = pm / Ops::nparty;
    const int64_t kbeg = (int64_t)split * k_per_split;
    const int64_t kend = min(ops.Kext, kbeg + k_per_split);
    T acc[NN];
#pragma unroll
    for (int j = 0; j < NN; ++j) acc[j] = 0;
    for (int64_t k = kbeg + lane; k < kend; k += 32) {
        T av = ops.a(p, m, k);
#pragma unroll
        for (int j = 0; j < NN; ++j)
            if (j < ops.N) acc[j] += av * ops.b(p, k, j);
    }
#pragma unroll
    for (int j = 0; j < NN; ++j) {
        if (j >= ops.N) break;
        T s = warp_sum<T>(acc[j]);
        if (lane == j) {
            if (partial == nullptr) ops.store(p, m, j, s);
            else {
                T *dst = partial + ((int64_t)p * ops.M + m) * ops.N + j;
                if (sizeof(T) == 8) atomicAdd((unsigned long long *)dst, (unsigned long long)s);
                else atomicAdd((unsigned int *)dst, (unsigned int)s);
            }
        }
    }
}

// Tall-skinny products (N <= NN = 16, short K'; the CNN conv im2col GEMMs, 100352 x 150 x 16):
// one thread per output row holding all N accumulators, the whole K' x N B operand staged in
// shared memory once per CTA (read as a broadcast), A gathered per (row, k) straight from the
// producers' buffers (consecutive rows = consecutive output pixels: coalesced).
template <typename T, class Ops, int NN>
__global__ void __launch_bounds__(256) ring_gemm_rows(Ops ops) {
    extern __shared__ __align__(16) unsigned char rows_smem[];
    T *Bs = reinterpret_cast<T *>(rows_smem);   // [Kext][NN]
    const int p = blockIdx.y;
    const int64_t Kx = ops.Kext;
    const int N = (int)ops.N;
    for (int64_t i = threadIdx.x; i < Kx * NN; i += blockDim.x) {
        const int64_t k = i / NN;
        const int n = (int)(i % NN);
        Bs[i] = n < N ? ops.b(p, k, n) : (T)0;
    }
    __syncthreads();
    const int64_t m = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (m >= ops.M) return;
    RingAcc<T> acc[NN];
#pragma unroll
    for (int j = 0; j < NN; ++j) acc[j].zero();
#pragma unroll 2
    for (int64_t k = 0; k < Kx; ++k) {
        const T a = ops.a(p, m, k);
        const T *b = Bs + k * NN;
#pragma unroll
        for (int j = 0; j < NN; ++j) acc[j].mac(a, b[j]);
    }
#pragma unroll
    for (int j = 0; j < NN; ++j)
        if (j < N) ops.store(p, m, j, acc[j].value());
}

template <typename T, class Ops>
__global__ void ring_gemm_finalize(Ops ops, const T *__restrict__ partial) {
    const int64_t total = ops.M * ops.N * Ops::nparty;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total;
         i += (int64_t)gridDim.x * blockDim.x) {
        int64_t p = i / (ops.M * ops.N), r = i - p * ops.M * ops.N;
        ops.store((int)p, r / ops.N, r % ops.N, partial[i]);
    }
}

}  // namespace psml
#include "gemm_cl.cuh"
#include "gemm_seg.cuh"
namespace psml {

// psml_options.simt_cluster = 0: route small products to the 16 x 16 one-output-per-thread kernel
// instead of the cluster split-K kernel (both bit-identical).
inline bool simt_cl_enabled() { return cur_opts().simt_cluster != 0; }

// psml_options.rows_kernel = 0 keeps tall-skinny products on the 16 x 16 small-tile kernel.
inline bool rows_kernel_enabled() { return cur_opts().rows_kernel != 0; }

// ---------------------------------------------------------------------------------------------
// host-side dispatcher: picks kernel, tile and split-K; `ws` must hold nparty*M*N words when
// split-K is chosen (ws_words reports the need; pass ws = nullptr to query).
// ---------------------------------------------------------------------------------------------
template <typename T, class Ops>
psml_status launch_ring_gemm(const Ops &ops, T *ws, int64_t ws_words, cudaStream_t stream,
                             int sm_count = 148) {
    const int64_t M = ops.M, N = ops.N, Kx = ops.Kext;
    if (M <= 0 || N <= 0) return PSML_OK;
    const int64_t outs = M * N * Ops::nparty;
    // split-K so the grid fills the GPU: ~2 CTAs (tiled) or ~16 warps (GEMV) per SM, each split
    // still >= 64 (tiled) / 256 (GEMV) deep.  Ring addition is exact, so partials are summed
    // with uint64/uint32 atomics and the epilogue runs once in ring_gemm_finalize.
    // kernel choice: warp-per-row GEMV for skinny outputs with few rows (w^T x, MLP output layer),
    // the 16 x 16 small-tile kernel for small outputs or skinny outputs with many rows (CNN conv
    // im2col GEMMs), the 64 x 64 register-blocked kernel otherwise.
    const bool gemv = N <= 2 && M * Ops::nparty <= 4096 && Kx <= 8192;
    // the cluster kernel splits K at most 8 ways: very deep products with few output tiles (the
    // CNN conv weight gradient, 75 x 200704 x 16) go to the small-tile kernel's deep split-K
    if (!gemv && M * N * Ops::nparty <= ((int64_t)1 << 19) && Kx <= 32768 && simt_cl_enabled()) {
        ProfScope prof(PROF_GEMM, stream, (double)M * N * Kx * Ops::nparty);
        return launch_ring_gemm_cl<T, Ops>(ops, stream, sm_count);
    }
    if (!gemv && N <= 16 && M * Ops::nparty >= 8192 && Kx * 16 * (int64_t)sizeof(T) <= 96 * 1024 &&
        rows_kernel_enabled()) {
        const size_t smem = (size_t)Kx * 16 * sizeof(T);
        static bool attr = false;   // per (T, Ops) instantiation
        if (!attr) {
            PSML_CUDA_TRY(cudaFuncSetAttribute(ring_gemm_rows<T, Ops, 16>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                               96 * 1024));
            attr = true;
        }
        ProfScope prof(PROF_GEMM, stream, (double)M * N * Kx * Ops::nparty);
        ring_gemm_rows<T, Ops, 16><<<dim3((unsigned)((M + 255) / 256), Ops::nparty), 256, smem, stream>>>(ops);
        PSML_LAUNCH_CHECK();
        return PSML_OK;
    }
    const bool small = !gemv && (N <= 16 || M * N * Ops::nparty <= ((int64_t)1 << 18));
    int splits = 1;
    if (small) {
        const int64_t tiles = ((M + 15) / 16) * ((N + 15) / 16) * Ops::nparty;
        const int64_t target = (int64_t)sm_count * (Kx >= 16384 ? 4 : 2);
        if (tiles < target && Kx > 512)
            splits = (int)std::max<int64_t>(1, std::min<int64_t>((target + tiles - 1) / tiles, Kx / 256));
    } else if (gemv) {
        const int64_t warps = M * Ops::nparty;
        const int64_t target = (int64_t)sm_count * 16;
        if (warps < target) splits = (int)std::max<int64_t>(1, std::min<int64_t>((target + warps - 1) / warps, Kx / 256));
    } else {
        const int64_t tiles = ((M + 63) / 64) * ((N + 63) / 64) * Ops::nparty;
        const int64_t target = (int64_t)sm_count * 2;
        if (tiles < target) splits = (int)std::max<int64_t>(1, std::min<int64_t>((target + tiles - 1) / tiles, Kx / 64));
    }
    if (splits > 1 && (ws == nullptr || ws_words < outs)) splits = 1;  // no workspace: no split
    T *partial = nullptr;
    if (splits > 1) {
        partial = ws;
        PSML_CUDA_TRY(cudaMemsetAsync(partial, 0, sizeof(T) * outs, stream));
    }
    int64_t kps = (Kx + splits - 1) / splits;
    ProfScope prof(PROF_GEMM, stream, (double)M * N * Kx * Ops::nparty);
    if (small) {
        kps = ((kps + 63) / 64) * 64;
        dim3 grid((unsigned)((N + 15) / 16), (unsigned)((M + 15) / 16), (unsigned)(Ops::nparty * splits));
        ring_gemm_small<T, Ops><<<grid, 256, 0, stream>>>(ops, kps, partial);
    } else if (gemv) {
        const int64_t warps = M * Ops::nparty * splits;
        const int blocks = (int)((warps * 32 + 255) / 256);
        if (N == 1) ring_gemv<T, 1, Ops><<<blocks, 256, 0, stream>>>(ops, kps, splits, partial);
        else if (N <= 2) ring_gemv<T, 2, Ops><<<blocks, 256, 0, stream>>>(ops, kps, splits, partial);
        else if (N <= 4) ring_gemv<T, 4, Ops><<<blocks, 256, 0, stream>>>(ops, kps, splits, partial);
        else if (N <= 8) ring_gemv<T, 8, Ops><<<blocks, 256, 0, stream>>>(ops, kps, splits, partial);
        else ring_gemv<T, 16, Ops><<<blocks, 256, 0, stream>>>(ops, kps, splits, partial);
    } else {
        kps = ((kps + 15) / 16) * 16;
        dim3 grid((unsigned)((N + 63) / 64), (unsigned)((M + 63) / 64), (unsigned)(Ops::nparty * splits));
        ring_gemm_tiled<T, 64, 64, 16, 4, 4, Ops><<<grid, 256, 0, stream>>>(ops, kps, partial);
    }
    PSML_LAUNCH_CHECK();
    if (splits > 1) {
        ring_gemm_finalize<T, Ops><<<grid_for(outs, 256), 256, 0, stream>>>(ops, partial);
        PSML_LAUNCH_CHECK();
    }
    return PSML_OK;
}

template <class Ops>
inline int64_t ring_gemm_ws_words(const Ops &ops) {
    return ops.M * ops.N * Ops::nparty;
}

}  // namespace psml
