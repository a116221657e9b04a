// engine.h -- internal declarations shared by engine.cu, model.cu and gemm_tc.cu.
#pragma once
#include <algorithm>
#include <initializer_list>

#include "ops.cuh"

namespace psml {

psml_status check_ring(psml_ring r);

// Peer-memory window of a connected peer transport for FUSED compute + exchange kernels (split
// deployment): this party's window (written by the peer), the peer's window (mapped), and the
// flag words -- an epoch counter and a done counter per call, one release/acquire flag per CTA.
constexpr int PW_MAX_CTAS = 64, PW_FLAG_STRIDE = 16, PW_EPOCH = 80, PW_DONE = 96, PW_FLAG_BASE = 128;
constexpr int64_t PW_BYTES = (int64_t)8 << 20;
struct PeerWindow {
    uint8_t *my_win, *peer_win;
    int64_t bytes;
    uint64_t *my_flags, *peer_flags;
};
bool xport_peer_window(psml_xport x, PeerWindow *w);   // false: not a connected peer transport
void xport_account(psml_xport x, int64_t exchanges, int64_t bytes);   // stats of fused exchanges
// run the rest of an ABI call with the options of ctx / model (null: defaults)
#define PSML_CTX_OPTS(c) ::psml::OptScope _psml_opts_((c) ? &reinterpret_cast<const ::psml::Ctx *>(c)->opts : nullptr)
psml_status check_ptrs(std::initializer_list<const void *> ps);
int current_sm_count();

struct Ctx {
    psml_ring ring{64, 13};
    int backend = 0;    // 0 auto, 1 CUDA-core, 2 tcgen05
    psml_options opts{0, 1, 0, 1, 1, 1, 1, 1, 1, 1, 0, 1, 1, 0, 1};   // = psml_options_default
    int sm_count = 148;
    bool tc_ok = false;
    void *ws = nullptr;
    size_t ws_bytes = 0;
    psml_status ensure_ws(size_t bytes);
    // per-party context (psml_ctx_create_party): this party, its pair transport, its DP group
    int party = -1;                 // -1: co-resident pair engine
    psml_xport xport = nullptr;
    psml_dp dp = nullptr;
    void *msg = nullptr;            // the party's send / receive message buffers
    size_t msg_bytes = 0;
    psml_status ensure_msg(size_t bytes);
    // tcgen05 limb GEMM pays once a party's product has >= 2^25 ring MACs (measured on B200:
    // 128x1568x128 is 2x faster on CUDA cores, 12544x256x64 1.5x and 1024^3 10x faster on tcgen05;
    // tools/mm_prof.py).
    bool use_tc(int64_t M, int64_t Kext, int64_t N) const {
        if (!tc_ok || backend == 1) return false;
        if (backend == 2) return true;
        return M >= 128 && N >= 64 && M * N * Kext >= ((int64_t)1 << 25);
    }
};

// ------------------------------------------------------------------------------------------------
// launch helpers (templates, used by engine.cu and model.cu)
// ------------------------------------------------------------------------------------------------
template <typename T>
psml_status hadamard_triplet_launch(const DealSeeds &S, uint64_t cid, int64_t n, void *const U[2], void *const V[2],
                                    void *const Z[2], cudaStream_t s, const uint32_t *step = nullptr) {
    Pair<T> u{{(T *)U[0], (T *)U[1]}}, v{{(T *)V[0], (T *)V[1]}}, z{{(T *)Z[0], (T *)Z[1]}};
    const int64_t nblk = (n + PerBlock<T>::value - 1) / PerBlock<T>::value;
    hadamard_triplet_kernel<T><<<grid_for(nblk, 128, 148 * 32), 128, 0, s>>>(
        dkey(S, TAG_U0, cid, step), dkey(S, TAG_U1, cid, step), dkey(S, TAG_V0, cid, step),
        dkey(S, TAG_V1, cid, step), dkey(S, TAG_Z0, cid, step), n, u, v, z);
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

template <typename T>
psml_status msb_dealer_launch(const DealSeeds &S, uint64_t cid, int64_t n, void *const mat[2], cudaStream_t s,
                              const uint32_t *step = nullptr) {
    const int L = ilog2_int(8 * (int)sizeof(T));
    const int64_t nblk = (n + PerBlock<T>::value - 1) / PerBlock<T>::value;
    dim3 grid((unsigned)grid_for(nblk, 128, 148 * 8), 4u);   // 3 AND groups + the daBit (R27)
    msb_dealer_kernel<T><<<grid, 128, 0, s>>>(S, cid, n, L, (T *)mat[0], (T *)mat[1], step);
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

// opened values for psml_trace: E = E_0 + E_1, F = F_0 + F_1 (from the trace's E_i/F_i copies)
template <typename T>
psml_status trace_opened(Ctx *c, int64_t M, int64_t K, int64_t N, const psml_trace *tr, cudaStream_t s) {
    (void)c;
    if (tr->E_open && tr->E[0] && tr->E[1]) {
        add_kernel<T><<<grid_for(M * K, 256), 256, 0, s>>>((const T *)tr->E[0], (const T *)tr->E[1], M * K, (T *)tr->E_open);
        PSML_LAUNCH_CHECK();
    }
    if (tr->F_open && tr->F[0] && tr->F[1]) {
        add_kernel<T><<<grid_for(K * N, 256), 256, 0, s>>>((const T *)tr->F[0], (const T *)tr->F[1], K * N, (T *)tr->F_open);
        PSML_LAUNCH_CHECK();
    }
    return PSML_OK;
}

psml_status tc_dealer_gemm(int l, const void *U0, const void *U1, const void *V0, const void *V1, int64_t M, int64_t K,
                           int64_t N, const void *Z0, void *Z1, void *ws, size_t ws_bytes, cudaStream_t s);

template <typename T>
size_t tc_beaver_ws_bytes(int64_t M, int64_t K, int64_t N);
template <typename T>
psml_status tc_beaver_matmul_ws(const T *const A[2], const T *const B[2], const T *const U[2], const T *const V[2],
                                const T *const Z[2], int64_t M, int64_t K, int64_t N, int flags, int trunc,
                                T *const C[2], void *ws, size_t ws_bytes, int sm_count, cudaStream_t s);

// Split-deployment round 2 on tcgen05 for one party (gemm_tc.cu).
psml_status tc_open_matmul_one(Ctx *c, int l, int party, const void *Es, const void *Er, const void *Fs,
                               const void *Fr, const void *U, const void *V, const void *Z, int64_t M, int64_t K,
                               int64_t N, int trunc, void *C, cudaStream_t s);

// tcgen05 Beaver product (gemm_tc.cu); PSML_ERR_UNSUPPORTED = take the CUDA-core path.
template <typename T>
psml_status tc_beaver_matmul(Ctx *c, const T *const A[2], const T *const B[2], const T *const U[2],
                             const T *const V[2], const T *const Z[2], int64_t M, int64_t K, int64_t N, int flags,
                             int trunc, T *const C[2], cudaStream_t s);

}  // namespace psml
