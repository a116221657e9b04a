// fused.cuh -- kernels of the fused co-resident training step (model.cu).
//
// Every Beaver product of the step reads opened operands E, X_1 = E + U_1 (A side) and F (B side)
// (gemm_seg.cuh).  Instead of one open launch per product, the kernel that PRODUCES an operand
// also opens it for its consumers -- it holds both parties' shares of the element anyway:
//   step start     weights (forward and transposed for gradin) and the input batch (forward and
//                  transposed for gradW_0): one multi-job open_list_kernel
//   ReLU chain     h_{l+1} -> A side of fwd_{l+1} and (transposed) of gradW_{l+1}
//   Eq. 9 chain    delta    -> B side of gradW_L and A side of gradin_L
//   backprop Had.  delta_l  -> B side of gradW_l and A side of gradin_l
// The opened values are exactly those of the stand-alone open pass (same ring sums), so the step
// stays bit-identical to the oracle (tested, and PSML_FUSE=0 runs the unfused step).
#pragma once
#include "kernels.cuh"

namespace psml {

// both parties in one thread
template <typename T>
__device__ __forceinline__ void emit_both(const Emits<T> &es, int64_t e, T v0, T v1) {
#pragma unroll
    for (int q = 0; q < 2; ++q) {
        if (q >= es.n) break;
        const Emit<T> &em = es.e[q];
        const int64_t di = emit_index(em, e);
        const T m0 = em.M[0][di], m1 = em.M[1][di];
        const T E = (T)(v0 - m0) + (T)(v1 - m1);
        em.E[di] = E;
        if (em.X1) em.X1[di] = E + m1;
    }
}

// ---------------------------------------------------------------------------------------------
// step-start opens: up to OPEN_MAX_JOBS OpenJobs (gemm_seg.cuh) in one launch, 32 x 32 tiles
// ---------------------------------------------------------------------------------------------
constexpr int OPEN_MAX_JOBS = 16;
template <typename T>
struct OpenList {
    OpenJob<T> j[OPEN_MAX_JOBS];
    int64_t tile_begin[OPEN_MAX_JOBS + 1];
    int n;
};

template <typename T>
__global__ void __launch_bounds__(256) open_list_kernel(const __grid_constant__ OpenList<T> L) {
    pdl_trigger();
    pdl_wait();
    __shared__ T tile[2][32][33];
    const int64_t t = blockIdx.x;
    int q = 0;
    for (int i = 1; i < L.n; ++i)
        if (t >= L.tile_begin[i]) q = i;
    const OpenJob<T> &J = L.j[q];
    const int64_t tt = t - L.tile_begin[q];
    const int64_t tiles_c = (J.cols + 31) / 32;
    const int64_t r0 = (tt / tiles_c) * 32, c0 = (tt % tiles_c) * 32;
    const int tx = threadIdx.x, ty = threadIdx.y;   // 32 x 8
    T s[2][4];
    if (J.trans) {
#pragma unroll
        for (int p = 0; p < 2; ++p)
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                const int i = ty + 8 * u;
                const int64_t sc = c0 + i, sr = r0 + tx;
                const int64_t scc = sc < J.cols ? sc : J.cols - 1, src = sr < J.rows ? sr : J.rows - 1;
                tile[p][i][tx] = J.src[p][scc * J.rows + src];
            }
        __syncthreads();
#pragma unroll
        for (int p = 0; p < 2; ++p)
#pragma unroll
            for (int u = 0; u < 4; ++u) s[p][u] = tile[p][tx][ty + 8 * u];
    } else {
#pragma unroll
        for (int p = 0; p < 2; ++p)
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                const int64_t r = r0 + ty + 8 * u, c = c0 + tx;
                s[p][u] = J.src[p][(r < J.rows ? r : J.rows - 1) * J.cols + (c < J.cols ? c : J.cols - 1)];
            }
    }
    T mk[2][4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
        const int64_t r = r0 + ty + 8 * u, c = c0 + tx;
        const int64_t o = (r < J.rows ? r : J.rows - 1) * J.cols + (c < J.cols ? c : J.cols - 1);
        mk[0][u] = J.mask[0][o];
        mk[1][u] = J.mask[1][o];
    }
#pragma unroll
    for (int u = 0; u < 4; ++u) {
        const int64_t r = r0 + ty + 8 * u, c = c0 + tx;
        if (r < J.rows && c < J.cols) {
            const int64_t o = r * J.cols + c;
            const T e = (T)(s[0][u] - mk[0][u]) + (T)(s[1][u] - mk[1][u]);
            J.open[o] = e;
            if (J.x) J.x[o] = (T)(J.scale * e + mk[1][u]);   // X_1 = E + U_1
        }
    }
}

// ---------------------------------------------------------------------------------------------
// backprop Hadamard (co-resident, both parties per thread): c = a (.) b with the Beaver triplet
// (U, V, Z), mask and open in one pass (Eqs. 4-5 elementwise), then the consumer opens of c
// ---------------------------------------------------------------------------------------------
template <typename T>
struct HadFused {
    const T *a[2], *b[2], *U[2], *V[2], *Z[2];
    T *c[2];
    int64_t n;
    Emits<T> em;
};

template <typename T>
__global__ void __launch_bounds__(256) had_fused_kernel(const __grid_constant__ HadFused<T> h) {
    pdl_trigger();
    // the Hadamard triplet of the first element is dealer material (complete before any PDL
    // predecessor started, see msb_chain_pair_kernel): load it before griddepcontrol.wait
    const int64_t i0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    T pu0 = 0, pu1 = 0, pv0 = 0, pv1 = 0;
    if (i0 < h.n) { pu0 = h.U[0][i0]; pu1 = h.U[1][i0]; pv0 = h.V[0][i0]; pv1 = h.V[1][i0]; }
    pdl_wait();
    for (int64_t i = i0; i < h.n; i += (int64_t)gridDim.x * blockDim.x) {
        const bool first = i == i0;
        const T u0 = first ? pu0 : h.U[0][i], u1 = first ? pu1 : h.U[1][i];
        const T v0 = first ? pv0 : h.V[0][i], v1 = first ? pv1 : h.V[1][i];
        const T E = (T)(h.a[0][i] - u0) + (T)(h.a[1][i] - u1);
        const T F = (T)(h.b[0][i] - v0) + (T)(h.b[1][i] - v1);
        const T c0 = E * v0 + u0 * F + h.Z[0][i];
        const T c1 = E * F + E * v1 + u1 * F + h.Z[1][i];
        if (h.c[0]) { h.c[0][i] = c0; h.c[1][i] = c1; }
        emit_both(h.em, i, c0, c1);
    }
}

// linear regression output: yhat = z, delta = z - Y, consumer opens of delta
template <typename T>
struct DeltaFused {
    const T *z[2], *Y[2];
    T *yhat[2], *delta[2];
    int64_t n;
    Emits<T> em;
};

template <typename T>
__global__ void __launch_bounds__(256) delta_fused_kernel(const __grid_constant__ DeltaFused<T> d) {
    pdl_trigger();
    pdl_wait();
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < d.n; i += (int64_t)gridDim.x * blockDim.x) {
        const T z0 = d.z[0][i], z1 = d.z[1][i];
        const T d0 = z0 - d.Y[0][i], d1 = z1 - d.Y[1][i];
        d.yhat[0][i] = z0; d.yhat[1][i] = z1;
        d.delta[0][i] = d0; d.delta[1][i] = d1;
        emit_both(d.em, i, d0, d1);
    }
}

// ---------------------------------------------------------------------------------------------
// SGD update of every layer in one launch (same arithmetic as update_kernel, R14)
// ---------------------------------------------------------------------------------------------
constexpr int UPD_MAX_LAYERS = 8;
template <typename T>
struct UpdateAll {
    T *Wm[UPD_MAX_LAYERS][2], *W[UPD_MAX_LAYERS][2];
    const T *g[UPD_MAX_LAYERS][2];
    int64_t begin[UPD_MAX_LAYERS + 1];
    int nl, s_grad, s_fwd[UPD_MAX_LAYERS];
    int wd;   // weight-decay shift (0 = none; SVM, R24)
};

template <typename T>
__global__ void __launch_bounds__(256) update_all_kernel(const __grid_constant__ UpdateAll<T> u) {
    pdl_trigger();
    pdl_wait();
    const int64_t total = u.begin[u.nl];
    for (int64_t x = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; x < total; x += (int64_t)gridDim.x * blockDim.x) {
        int l = 0;
        for (int q = 1; q < u.nl; ++q)
            if (x >= u.begin[q]) l = q;
        const int64_t i = x - u.begin[l];
#pragma unroll
        for (int p = 0; p < 2; ++p) {
            const T old = u.Wm[l][p][i];
            const T dec = u.wd ? trunc_share<T>(old, p, u.wd) : (T)0;
            const T wm = old - (trunc_share<T>(u.g[l][p][i], p, u.s_grad) + dec);
            u.Wm[l][p][i] = wm;
            u.W[l][p][i] = trunc_share<T>(wm, p, u.s_fwd[l]);
        }
    }
}

}  // namespace psml
