// ops.cuh -- host-side building blocks of the co-resident pair engine (shared by engine.cu).
// Each op = the sequence of round kernels of one protocol step, with explicit workspaces so a
// model step allocates nothing (and can be captured in a CUDA graph).
#pragma once
#include <algorithm>
#include <cstdlib>

#include "common.cuh"
#include "gemm_simt.cuh"
#include "kernels.cuh"

namespace psml {

constexpr int EW_THREADS = 256;

// MSB chain execution: 0 = one launch running each element through every round in order,
// 1 = one kernel per round (psml_options.msb_chain; tests compare both).
inline int chain_mode() { return cur_opts().msb_chain; }

inline int ew_grid(int64_t n) { return grid_for(n, EW_THREADS, 148 * 32); }

// Tensor-core limb GEMM entry (gemm_tc.cu).  Returns PSML_ERR_UNSUPPORTED when the shape or
// device does not take the tcgen05 path (the caller then uses the CUDA-core kernels).
struct TcBeaverArgs;
psml_status tc_ring_gemm_plain(int l, const void *A, const void *B, int64_t M, int64_t K, int64_t N,
                               void *C, void *ws, size_t ws_bytes, cudaStream_t s);
size_t tc_ring_gemm_ws_bytes(int l, int64_t M, int64_t K, int64_t N);
bool tc_available();

// ---------------------------------------------------------------------------------------------
// Beaver matmul: mask round (Eq. 4) + fused open/Eq. 8 GEMM/epilogue round.
// ws_words needs: M*K*2 + K*N*2 (messages) + 2*M*N (split-K partials).
// ---------------------------------------------------------------------------------------------
template <typename T>
inline int64_t beaver_ws_words(int64_t M, int64_t K, int64_t N) {
    return 2 * M * K + 2 * K * N + 2 * M * N;
}

template <typename T>
psml_status beaver_matmul(const T *const A[2], const T *const B[2], const T *const U[2],
                          const T *const V[2], const T *const Z[2], int64_t M, int64_t K,
                          int64_t N, int flags, int trunc, T *const C[2], T *ws, int64_t ws_words,
                          cudaStream_t s, int sm_count, T *const traceE[2] = nullptr,
                          T *const traceF[2] = nullptr) {
    const int tA = (flags & PSML_TRANS_A) ? 1 : 0, tB = (flags & PSML_TRANS_B) ? 1 : 0;
    if (!(flags & PSML_PAPER_FORM) && seg_eligible(M, K, N, 2) && simt_cl_enabled()) {
        // open once (E, X_1 = E + U_1, F), then C_p = [X_p | E] . [F ; V_p] + Z_p (gemm_seg.cuh)
        T *E = ws, *X1 = ws + M * K, *F = ws + 2 * M * K;
        OpenJobs<T> oj;
        oj.j[0] = {{A[0], A[1]}, {U[0], U[1]}, E, X1, U[1], (T)1, M, K, tA};
        oj.j[1] = {{B[0], B[1]}, {V[0], V[1]}, F, nullptr, nullptr, (T)0, K, N, tB};
        PSML_TRY(launch_open<T>(oj, s));
        const bool tE = traceE && traceE[0] && traceE[1], tF = traceF && traceF[0] && traceF[1];
        if (tE || tF) {   // the parties' masked messages E_i, F_i for the trace (tests only)
            MaskJobs<T> tj;
            tj.j[0] = {A[0], U[0], tE ? traceE[0] : nullptr, M, K, tA};
            tj.j[1] = {A[1], U[1], tE ? traceE[1] : nullptr, M, K, tA};
            tj.j[2] = {B[0], V[0], tF ? traceF[0] : nullptr, K, N, tB};
            tj.j[3] = {B[1], V[1], tF ? traceF[1] : nullptr, K, N, tB};
            const int first = tE ? 0 : 2, count = (tE ? 2 : 0) + (tF ? 2 : 0);
            for (int q = 0; q < count; ++q) tj.j[q] = tj.j[first + q];
            tj.count = count;
            const int64_t maxt = std::max(((M + 31) / 32) * ((K + 31) / 32), ((K + 31) / 32) * ((N + 31) / 32));
            mask_kernel<T><<<dim3((unsigned)std::min<int64_t>(maxt, 148 * 8), 1, (unsigned)count), dim3(32, 8), 0, s>>>(tj);
            PSML_LAUNCH_CHECK();
        }
        SegArgs<T> sa{};
        sa.X[0] = U[0]; sa.X[1] = X1; sa.E = E; sa.F = F;
        for (int p = 0; p < 2; ++p) { sa.V[p] = V[p]; sa.Z[p] = Z[p]; sa.C[p] = C[p]; sa.party[p] = p; }
        sa.M = M; sa.N = N; sa.K = K; sa.trunc = trunc;
        return launch_seg_gemm<T>(sa, 2, s, sm_count);
    }
    T *mE0 = ws, *mE1 = ws + M * K, *mF0 = ws + 2 * M * K, *mF1 = mF0 + K * N;
    T *partial = mF1 + K * N;
    MaskJobs<T> jobs;
    jobs.j[0] = {A[0], U[0], mE0, M, K, tA};
    jobs.j[1] = {A[1], U[1], mE1, M, K, tA};
    jobs.j[2] = {B[0], V[0], mF0, K, N, tB};
    jobs.j[3] = {B[1], V[1], mF1, K, N, tB};
    jobs.count = 4;
    const int64_t maxt = std::max(((M + 31) / 32) * ((K + 31) / 32), ((K + 31) / 32) * ((N + 31) / 32));
    {
        ProfScope prof(PROF_MASK, s, 3.0 * sizeof(T) * 2 * (M * K + K * N));
        mask_kernel<T><<<dim3((unsigned)std::min<int64_t>(maxt, 148 * 8), 1, 4), dim3(32, 8), 0, s>>>(jobs);
        PSML_LAUNCH_CHECK();
    }
    auto run = [&](auto ops) -> psml_status {
        using Ops = decltype(ops);
        ops.mE0 = mE0; ops.mE1 = mE1; ops.mF0 = mF0; ops.mF1 = mF1;
        for (int p = 0; p < 2; ++p) {
            ops.U[p] = U[p]; ops.V[p] = V[p]; ops.Z[p] = Z[p]; ops.A[p] = A[p]; ops.B[p] = B[p]; ops.C[p] = C[p];
        }
        ops.M = M; ops.N = N; ops.K = K; ops.Kext = 2 * K;
        ops.transA = tA; ops.transB = tB; ops.trunc = trunc;
        return launch_ring_gemm<T, Ops>(ops, partial, ws_words - (partial - ws), s, sm_count);
    };
    if (flags & PSML_PAPER_FORM) PSML_TRY(run(BeaverOps<T, 1>{}));
    else PSML_TRY(run(BeaverOps<T, 0>{}));
    if (traceE) {
        for (int p = 0; p < 2; ++p)
            if (traceE[p]) PSML_CUDA_TRY(cudaMemcpyAsync(traceE[p], p ? mE1 : mE0, sizeof(T) * M * K, cudaMemcpyDeviceToDevice, s));
    }
    if (traceF) {
        for (int p = 0; p < 2; ++p)
            if (traceF[p]) PSML_CUDA_TRY(cudaMemcpyAsync(traceF[p], p ? mF1 : mF0, sizeof(T) * K * N, cudaMemcpyDeviceToDevice, s));
    }
    return PSML_OK;
}

// Co-resident Beaver matmul with the mask round fused into the GEMM's operand loads (one launch;
// bit-identical to beaver_matmul).  ws: 2*M*N words for split-K partials.
template <typename T>
psml_status beaver_matmul_fused(const T *const A[2], const T *const B[2], const T *const U[2],
                                const T *const V[2], const T *const Z[2], int64_t M, int64_t K,
                                int64_t N, int flags, int trunc, T *const C[2], T *ws, int64_t ws_words,
                                cudaStream_t s, int sm_count) {
    BeaverFusedOps<T> ops;
    for (int p = 0; p < 2; ++p) {
        ops.A[p] = A[p]; ops.B[p] = B[p]; ops.U[p] = U[p]; ops.V[p] = V[p]; ops.Z[p] = Z[p]; ops.C[p] = C[p];
    }
    ops.M = M; ops.N = N; ops.K = K; ops.Kext = 2 * K;
    ops.transA = (flags & PSML_TRANS_A) ? 1 : 0;
    ops.transB = (flags & PSML_TRANS_B) ? 1 : 0;
    ops.trunc = trunc;
    return launch_ring_gemm<T, BeaverFusedOps<T>>(ops, ws, ws_words, s, sm_count);
}

// ---------------------------------------------------------------------------------------------
// Convolution Beaver product (im2col ring GEMM, mask on the raw input; R17)
// transposed = 0: C = im2col(X) . Wc         M = B*OH*OW, K = C*k*k,  N = Cout
// transposed = 1: C = im2col(X)^T . D        M = C*k*k,   K = B*OH*OW, N = Cout
// ws: 2*nin (raw-input messages) + 2*K*N (F messages) + 2*M*N (split-K)
// ---------------------------------------------------------------------------------------------
// Conv weight gradient (the transposed conv product, untruncated: R17 and a9), per image:
//   C_p[m][n] = Z_p[m][n] + sum_b sum_(oy,ox) (p E + U_p)[b, src(m) + oy W + ox] F[(b,oy,ox)][n]
//                                           +  E[b, src(m) + oy W + ox]        V_p[(b,oy,ox)][n]
// with E = mE0 + mE1 and F = mF0 + mF1 (the opened messages) and src(m) = coloff[m], m = (ch, ky,
// kx) -- the same sum as ConvBeaverOps with transposed = 1, regrouped by image.  One CTA = one
// (image, party, half of the output rows): the image's operand plane and the half's F (or V) rows
// sit in shared memory, thread (m, n-quad) runs its 4 split accumulators over the half's output
// positions, and the partial tile is added to C_p (pre-set to Z_p) with 64-bit atomics (ring
// addition is exact, so the order does not matter: bit-identical to the generic GEMM, tested).
template <typename T>
__global__ void __launch_bounds__(1024) conv_gw_image_kernel(const T *__restrict__ mE0, const T *__restrict__ mE1,
                                                             const T *__restrict__ U0, const T *__restrict__ U1,
                                                             const T *__restrict__ mF0, const T *__restrict__ mF1,
                                                             const T *__restrict__ V0, const T *__restrict__ V1,
                                                             ConvGeom g, int64_t N, T *C0, T *C1) {
    extern __shared__ __align__(16) unsigned char conv_smem[];
    T *img = (T *)conv_smem;
    const int chw = g.C * g.H * g.W;
    const int b = blockIdx.x, p = blockIdx.y, half = blockIdx.z;
    const int oy0 = half * ((g.OH + 1) / 2), oy1 = min(g.OH, oy0 + (g.OH + 1) / 2);
    const int npos = (oy1 - oy0) * g.OW;
    T *fb = img + chw;
    const int M = g.C * g.k * g.k, NQ = (int)N / 4;
    const int t = threadIdx.x;
    const bool act = t < M * NQ;
    const int m = act ? t % M : 0, nq = act ? t / M : 0;
    const int off = act ? g.coloff[m] : 0;
    RingAcc<T> acc[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) acc[j].zero();
    const T *ub = (p ? U1 : U0) + (int64_t)b * chw;
    const T *vb = (p ? V1 : V0);
    const int64_t r0 = (int64_t)b * g.OH * g.OW + (int64_t)oy0 * g.OW;   // first im2col row of the half
    for (int seg = 0; seg < 2; ++seg) {
        // operand plane: segment 0 -> p E + U_p, segment 1 -> E; rows: segment 0 -> F, 1 -> V_p
        for (int i = t; i < chw; i += blockDim.x) {
            const int64_t gi = (int64_t)b * chw + i;
            const T e = mE0[gi] + mE1[gi];
            img[i] = seg == 0 ? (T)((T)p * e + ub[i]) : e;
        }
        for (int i = t; i < npos * (int)N; i += blockDim.x) {
            const int64_t gi = r0 * N + i;
            fb[i] = seg == 0 ? (T)(mF0[gi] + mF1[gi]) : vb[gi];
        }
        __syncthreads();
        if (act) {
            for (int oy = oy0; oy < oy1; ++oy) {
                const T *arow = img + off + oy * g.W;
                const T *brow = fb + (int64_t)(oy - oy0) * g.OW * N + 4 * nq;
#pragma unroll 4
                for (int ox = 0; ox < g.OW; ++ox) {
                    const T a = arow[ox];
                    const ulonglong2 b01 = *(const ulonglong2 *)(brow + ox * N);
                    const ulonglong2 b23 = *(const ulonglong2 *)(brow + ox * N + 2);
                    acc[0].mac(a, (T)b01.x); acc[1].mac(a, (T)b01.y);
                    acc[2].mac(a, (T)b23.x); acc[3].mac(a, (T)b23.y);
                }
            }
        }
        __syncthreads();
    }
    if (act) {
        T *c = (p ? C1 : C0) + (int64_t)m * N + 4 * nq;
#pragma unroll
        for (int j = 0; j < 4; ++j) atomicAdd((unsigned long long *)(c + j), (unsigned long long)acc[j].value());
    }
}

// psml_options.conv_gw = 0 keeps the weight gradient on the generic im2col GEMM (tests)
inline bool conv_gw_enabled() { return cur_opts().conv_gw != 0; }

// The fast path applies to the untruncated weight gradient in Z_2^64 with N % 4 == 0 and
// operands that fit shared memory; false -> the generic im2col GEMM.
template <typename T>
bool conv_gw_fast_ok(const ConvGeom &g, int64_t N, int transposed, int trunc) {
    if (sizeof(T) != 8 || !transposed || trunc != 0 || N % 4 != 0) return false;
    const int64_t M = (int64_t)g.C * g.k * g.k;
    if (M * (N / 4) > 1024) return false;
    const int64_t words = (int64_t)g.C * g.H * g.W + (int64_t)((g.OH + 1) / 2) * g.OW * N;
    return words * (int64_t)sizeof(T) <= 200 * 1024;
}

template <typename T>
psml_status conv_gw_fast(const T *mE0, const T *mE1, const T *const UX[2], const T *mF0, const T *mF1,
                         const T *const V[2], const T *const Z[2], int64_t batch, const ConvGeom &g, int64_t N,
                         T *const C[2], cudaStream_t s) {
    const int64_t M = (int64_t)g.C * g.k * g.k;
    for (int p = 0; p < 2; ++p)
        PSML_CUDA_TRY(cudaMemcpyAsync(C[p], Z[p], sizeof(T) * (size_t)(M * N), cudaMemcpyDeviceToDevice, s));
    const size_t smem = sizeof(T) * (size_t)((int64_t)g.C * g.H * g.W + (int64_t)((g.OH + 1) / 2) * g.OW * N);
    static bool attr = false;
    if (!attr) {
        PSML_CUDA_TRY(cudaFuncSetAttribute(conv_gw_image_kernel<T>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                           200 * 1024));
        attr = true;
    }
    const int threads = (int)((M * (N / 4) + 31) / 32 * 32);
    conv_gw_image_kernel<T><<<dim3((unsigned)batch, 2, 2), threads, smem, s>>>(mE0, mE1, UX[0], UX[1], mF0, mF1,
                                                                               V[0], V[1], g, N, C[0], C[1]);
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

template <typename T>
psml_status conv_beaver(const T *const X[2], const T *const Bm[2], const T *const UX[2],
                        const T *const V[2], const T *const Z[2], int64_t batch, ConvGeom g,
                        int transposed, int64_t N, int trunc, T *const C[2], T *ws, int64_t ws_words,
                        cudaStream_t s, int sm_count) {
    const int64_t nin = batch * g.C * g.H * g.W;
    const int64_t rows = batch * g.OH * g.OW, kk = (int64_t)g.C * g.k * g.k;
    const int64_t M = transposed ? kk : rows, K = transposed ? rows : kk;
    T *mE0 = ws, *mE1 = ws + nin, *mF0 = ws + 2 * nin, *mF1 = mF0 + K * N, *partial = mF1 + K * N;
    MaskJobs<T> jobs;
    jobs.j[0] = {X[0], UX[0], mE0, batch, (int64_t)g.C * g.H * g.W, 0};
    jobs.j[1] = {X[1], UX[1], mE1, batch, (int64_t)g.C * g.H * g.W, 0};
    jobs.j[2] = {Bm[0], V[0], mF0, K, N, 0};
    jobs.j[3] = {Bm[1], V[1], mF1, K, N, 0};
    jobs.count = 4;
    const int64_t maxt = std::max(((batch + 31) / 32) * (((int64_t)g.C * g.H * g.W + 31) / 32), ((K + 31) / 32) * ((N + 31) / 32));
    mask_kernel<T><<<dim3((unsigned)std::min<int64_t>(maxt, 148 * 8), 1, 4), dim3(32, 8), 0, s>>>(jobs);
    PSML_LAUNCH_CHECK();
    if (conv_gw_fast_ok<T>(g, N, transposed, trunc) && conv_gw_enabled())
        return conv_gw_fast<T>(mE0, mE1, UX, mF0, mF1, V, Z, batch, g, N, C, s);
    ConvBeaverOps<T> ops;
    ops.mE0 = mE0; ops.mE1 = mE1; ops.mF0 = mF0; ops.mF1 = mF1;
    for (int p = 0; p < 2; ++p) { ops.UX[p] = UX[p]; ops.V[p] = V[p]; ops.Z[p] = Z[p]; ops.C[p] = C[p]; }
    ops.g = g; ops.M = M; ops.N = N; ops.K = K; ops.Kext = 2 * K; ops.transposed = transposed; ops.trunc = trunc;
    return launch_ring_gemm<T, ConvBeaverOps<T>>(ops, partial, ws_words - (partial - ws), s, sm_count);
}

// Split deployment, one party: round 1 writes this party's messages (E_send over the un-expanded
// input, F_send); the caller exchanges them; round 2 opens them inside the im2col GEMM.
template <typename T>
psml_status conv_mask_party(const T *X, const T *Bm, const T *UX, const T *V, int64_t batch, ConvGeom g, int64_t K,
                            int64_t N, T *Es, T *Fs, cudaStream_t s) {
    MaskJobs<T> jobs;
    jobs.j[0] = {X, UX, Es, batch, (int64_t)g.C * g.H * g.W, 0};
    jobs.j[1] = {Bm, V, Fs, K, N, 0};
    jobs.count = 2;
    const int64_t maxt = std::max(((batch + 31) / 32) * (((int64_t)g.C * g.H * g.W + 31) / 32), ((K + 31) / 32) * ((N + 31) / 32));
    mask_kernel<T><<<dim3((unsigned)std::min<int64_t>(maxt, 148 * 8), 1, 2), dim3(32, 8), 0, s>>>(jobs);
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

template <typename T>
psml_status conv_open_party(int party, const T *Es, const T *Er, const T *Fs, const T *Fr, const T *UX, const T *V,
                            const T *Z, int64_t batch, ConvGeom g, int transposed, int64_t N, int trunc, T *C,
                            T *partial, int64_t partial_words, cudaStream_t s, int sm_count) {
    const int64_t rows = batch * g.OH * g.OW, kk = (int64_t)g.C * g.k * g.k;
    ConvBeaverOps1<T> ops;
    ops.mE0 = Es; ops.mE1 = Er; ops.mF0 = Fs; ops.mF1 = Fr; ops.UX = UX; ops.V = V; ops.Z = Z; ops.C = C;
    ops.g = g; ops.M = transposed ? kk : rows; ops.N = N; ops.K = transposed ? rows : kk; ops.Kext = 2 * ops.K;
    ops.transposed = transposed; ops.trunc = trunc; ops.party = party;
    return launch_ring_gemm<T, ConvBeaverOps1<T>>(ops, partial, partial_words, s, sm_count);
}

template <typename T>
inline int64_t conv_ws_words(int64_t batch, ConvGeom g, int transposed, int64_t N) {
    const int64_t nin = batch * g.C * g.H * g.W;
    const int64_t rows = batch * g.OH * g.OW, kk = (int64_t)g.C * g.k * g.k;
    const int64_t M = transposed ? kk : rows, K = transposed ? rows : kk;
    return 2 * nin + 2 * K * N + 2 * M * N;
}

// ---------------------------------------------------------------------------------------------
// Hadamard (2 rounds).  ws: 4 n words.
// ---------------------------------------------------------------------------------------------
template <typename T>
psml_status beaver_hadamard(const T *const A[2], const T *const B[2], const T *const U[2],
                            const T *const V[2], const T *const Z[2], int64_t n, int trunc,
                            T *const C[2], T *ws, cudaStream_t s) {
    Pair<T> mE{{ws, ws + n}}, mF{{ws + 2 * n, ws + 3 * n}};
    // algorithmic bytes: round 1 reads A,B,U,V writes E,F (6 words/party); round 2 reads
    // E_0,E_1,F_0,F_1,U,V,Z writes C (4 + 4 per party)
    ProfScope prof(PROF_HAD, s, (double)sizeof(T) * n * (12 + 12));
    CPair<T> a{{A[0], A[1]}}, b{{B[0], B[1]}}, u{{U[0], U[1]}}, v{{V[0], V[1]}}, z{{Z[0], Z[1]}};
    hadamard_mask_kernel<T><<<ew_grid(n), EW_THREADS, 0, s>>>(a, b, u, v, n, mE, mF);
    PSML_LAUNCH_CHECK();
    CPair<T> ce{{mE.p[0], mE.p[1]}}, cf{{mF.p[0], mF.p[1]}};
    hadamard_open_kernel<T><<<ew_grid(n), EW_THREADS, 0, s>>>(ce, cf, u, v, z, n, trunc, Pair<T>{{C[0], C[1]}});
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

// ---------------------------------------------------------------------------------------------
// MSB chain and the activations built on it.  ws: 6 n words per party (G, P, 4 msg) = 12 n.
// what: 0 = msb only (msbA), 1 = ReLU (y = x . drelu), 2 = Eq. 9 (x given as z of n/2; y of n/2,
//       optional delta = y - Ysub).
// ---------------------------------------------------------------------------------------------
template <typename T>
inline int64_t msb_ws_words(int64_t n) { return 12 * n; }

template <typename T>
psml_status msb_chain(const T *const x[2], int64_t n, const T *const mat[2], int mode, T half,
                      int what, T *const msbA[2], T *const msbB[2], T *const drelu[2],
                      const T *const U[2], const T *const V[2], const T *const Z[2], T *const y[2],
                      const T *const Ysub[2], T *const delta[2], T *ws, cudaStream_t s,
                      const Emits<T> *em = nullptr) {
    const int l = 8 * (int)sizeof(T);
    if (em && em->n && chain_mode() != 0) return fail(PSML_ERR_UNSUPPORTED, "operand emits need the lane-pair chain");
    MsbArgs<T> a;
    a.x = CPair<T>{{x[0], x[1]}};
    a.mat = CPair<T>{{mat[0], mat[1]}};
    a.G = Pair<T>{{ws, ws + n}};
    a.P = Pair<T>{{ws + 2 * n, ws + 3 * n}};
    a.msg = Pair<T>{{ws + 4 * n, ws + 8 * n}};
    a.n = n; a.mode = mode; a.half = half; a.L = ilog2_int(l); a.l = l;
    // algorithmic bytes of the chain (both parties): per AND round each party reads 2 message
    // words of both parties + 3 material words + state and writes state + 2 messages
    ProfScope prof(PROF_MSB, s, (double)sizeof(T) * n * (2.0 * (a.L + 2) * 14 + 16));
    Pair<T> mE{{a.msg.p[0] + n, a.msg.p[1] + n}}, mF{{a.msg.p[0] + 2 * n, a.msg.p[1] + 2 * n}};
    ChainOut<T> o;
    o.msbA = Pair<T>{{msbA ? msbA[0] : nullptr, msbA ? msbA[1] : nullptr}};
    o.msbB = Pair<T>{{msbB ? msbB[0] : nullptr, msbB ? msbB[1] : nullptr}};
    o.drelu = Pair<T>{{drelu ? drelu[0] : nullptr, drelu ? drelu[1] : nullptr}};
    o.y = Pair<T>{{y ? y[0] : nullptr, y ? y[1] : nullptr}};
    o.delta = Pair<T>{{delta ? delta[0] : nullptr, delta ? delta[1] : nullptr}};
    o.U = CPair<T>{{U ? U[0] : nullptr, U ? U[1] : nullptr}};
    o.V = CPair<T>{{V ? V[0] : nullptr, V ? V[1] : nullptr}};
    o.Z = CPair<T>{{Z ? Z[0] : nullptr, Z ? Z[1] : nullptr}};
    o.Ysub = CPair<T>{{Ysub ? Ysub[0] : nullptr, Ysub ? Ysub[1] : nullptr}};
    o.mE = mE;
    o.mF = mF;
    o.what = what;
    o.em.n = 0;
    if (em) o.em = *em;
    if (chain_mode() == 0) {   // one launch; lane pair = (party 0, party 1) of one element
        const int tpb = EW_THREADS;
        const int64_t threads = what == 2 ? ((n / 2 + 7) / 8) * 32 : 2 * n;
        const int blocks = (int)((threads + tpb - 1) / tpb);
        cudaError_t e;
        if (what == 0) e = launch_pdl(msb_chain_pair_kernel<T, 0>, dim3(blocks), dim3(tpb), s, a, o);
        else if (what == 1) e = launch_pdl(msb_chain_pair_kernel<T, 1>, dim3(blocks), dim3(tpb), s, a, o);
        else e = launch_pdl(msb_chain_pair_kernel<T, 2>, dim3(blocks), dim3(tpb), s, a, o);
        if (e != cudaSuccess) return fail(PSML_ERR_CUDA, std::string("msb chain launch: ") + cudaGetErrorString(e));
        PSML_LAUNCH_CHECK();
        return PSML_OK;
    }
    const int g = ew_grid(n);
    msb_round0_kernel<T><<<g, EW_THREADS, 0, s>>>(a);
    PSML_LAUNCH_CHECK();
    for (int j = 1; j <= a.L; ++j) {
        msb_level_kernel<T><<<g, EW_THREADS, 0, s>>>(a, j);
        PSML_LAUNCH_CHECK();
    }
    msb_final_kernel<T><<<g, EW_THREADS, 0, s>>>(a, o.msbB);
    PSML_LAUNCH_CHECK();
    msb_b2a_kernel<T><<<g, EW_THREADS, 0, s>>>(a, o.msbA, o.drelu, o.U, o.V, mE, mF, what == 0 ? 0 : 1);
    PSML_LAUNCH_CHECK();
    if (what == 0) return PSML_OK;
    CPair<T> ce{{mE.p[0], mE.p[1]}}, cf{{mF.p[0], mF.p[1]}};
    if (what == 1) {
        hadamard_open_kernel<T><<<g, EW_THREADS, 0, s>>>(ce, cf, o.U, o.V, o.Z, n, 0, o.y);
    } else {
        const int64_t nh = n / 2;
        eq9_open_kernel<T><<<ew_grid(nh), EW_THREADS, 0, s>>>(ce, cf, o.U, o.V, o.Z, nh, o.y, o.Ysub, o.delta);
    }
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

}  // namespace psml
