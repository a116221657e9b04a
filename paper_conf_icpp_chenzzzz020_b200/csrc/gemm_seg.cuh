// gemm_seg.cuh -- the opened Beaver product as a plain two-segment ring GEMM (Eq. 8,
// L175: the K-concatenation [i.E + U_i | E] . [F ; V_i]), for the small products of the training
// workloads.  Included by gemm_simt.cuh.
//
//   open_kernel   one pass over the masked messages: E = E_0 + E_1 (op(A) layout, M x K),
//                 X_1 = E + U_1 (the left segment of party 1; party 0's is U_0 itself) and
//                 F = F_0 + F_1 (K x N).  Co-resident: E_i = op(A_i) - U_i formed in the same
//                 pass (the mask round, Eq. 4); split deployment: E_send + E_recv (Eq. 5).
//   seg_gemm      C_p = [X_p | E] . [F ; V_p] + Z_p, truncated.  Every operand is a row-major
//                 matrix, so tiles stream into shared memory with element-wide cp.async (zero-filled
//                 at the ragged edges) through a 4-stage pipeline; 32 x 32 tile, 2 x 2 split
//                 accumulators per thread, K split over a (1, 1, ks) cluster and reduced through
//                 DSMEM by cl_finish (gemm_cl.cuh).
// Same ring arithmetic as the BeaverOps loaders (bit-identical, tested).
#pragma once
#include "common.cuh"

namespace psml {

// ---------------------------------------------------------------------------------------------
// open kernel: job 0 = A side (E, X_1), job 1 = B side (F).  Sources are either the parties'
// inputs with masks (co-resident: E = (op(src_0) - mask_0) + (op(src_1) - mask_1)) or two
// messages (split: E = msg_0 + msg_1, mask = nullptr).  X = party_scale.E + xmask when xmask set.
// ---------------------------------------------------------------------------------------------
template <typename T>
struct OpenJob {
    const T *src[2];   // op layout unless trans (then stored cols x rows)
    const T *mask[2];  // nullptr: sources are already masked messages (never transposed)
    T *open;           // rows x cols
    T *x;              // optional rows x cols: scale * open + xmask
    const T *xmask;
    T scale;
    int64_t rows, cols;
    int trans;
};
template <typename T> struct OpenJobs { OpenJob<T> j[2]; };

template <typename T>
__global__ void __launch_bounds__(256) open_kernel(OpenJobs<T> jobs) {
    __shared__ T tile[2][32][33];
    const OpenJob<T> J = jobs.j[blockIdx.z];
    const int64_t tiles_c = (J.cols + 31) / 32;
    const int64_t tiles = ((J.rows + 31) / 32) * tiles_c;
    const int tx = threadIdx.x, ty = threadIdx.y;   // 32 x 8
    for (int64_t t = blockIdx.x; t < tiles; t += gridDim.x) {
        const int64_t r0 = (t / tiles_c) * 32, c0 = (t % tiles_c) * 32;
        T s[2][4];
        if (J.trans) {   // src stored cols x rows: read coalesced along rows, transpose through smem
            __syncthreads();
#pragma unroll
            for (int q = 0; q < 2; ++q)
#pragma unroll
                for (int u = 0; u < 4; ++u) {
                    const int i = ty + 8 * u;
                    const int64_t sc = c0 + i, sr = r0 + tx;
                    const int64_t scc = sc < J.cols ? sc : J.cols - 1, src = sr < J.rows ? sr : J.rows - 1;
                    tile[q][i][tx] = J.src[q][scc * J.rows + src];
                }
            __syncthreads();
#pragma unroll
            for (int q = 0; q < 2; ++q)
#pragma unroll
                for (int u = 0; u < 4; ++u) s[q][u] = tile[q][tx][ty + 8 * u];
        } else {
#pragma unroll
            for (int q = 0; q < 2; ++q)
#pragma unroll
                for (int u = 0; u < 4; ++u) {
                    const int64_t r = r0 + ty + 8 * u, c = c0 + tx;
                    const int64_t o = (r < J.rows ? r : J.rows - 1) * J.cols + (c < J.cols ? c : J.cols - 1);
                    s[q][u] = J.src[q][o];
                }
        }
        T mk[2][4], xm[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            const int64_t r = r0 + ty + 8 * u, c = c0 + tx;
            const int64_t o = (r < J.rows ? r : J.rows - 1) * J.cols + (c < J.cols ? c : J.cols - 1);
            mk[0][u] = J.mask[0] ? J.mask[0][o] : (T)0;
            mk[1][u] = J.mask[1] ? J.mask[1][o] : (T)0;
            xm[u] = J.x ? J.xmask[o] : (T)0;
        }
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            const int64_t r = r0 + ty + 8 * u, c = c0 + tx;
            if (r < J.rows && c < J.cols) {
                const int64_t o = r * J.cols + c;
                const T e = (T)(s[0][u] - mk[0][u]) + (T)(s[1][u] - mk[1][u]);
                J.open[o] = e;
                if (J.x) J.x[o] = (T)(J.scale * e + xm[u]);
            }
        }
    }
}

// ---------------------------------------------------------------------------------------------
// two-segment GEMM, grouped: up to SEG_MAX_JOBS independent products (e.g. gradW_l and gradin_l,
// which consume the same delta) in one launch
// ---------------------------------------------------------------------------------------------
template <typename T>
struct SegArgs {
    const T *X[2];     // left segment per party (M x K)
    const T *E;        // right segment (M x K), shared
    const T *F;        // top segment (K x N), shared
    const T *V[2];     // bottom segment per party (K x N)
    const T *Z[2];
    T *C[2];
    int party[2];      // party index used by the truncation of slot p
    int64_t M, N, K;
    int trunc;
    int nparty;        // 1 (split deployment) or 2 (co-resident)
};

constexpr int SEG_MAX_JOBS = 4;
template <typename T>
struct SegGroup {
    SegArgs<T> j[SEG_MAX_JOBS];
    int64_t tile_begin[SEG_MAX_JOBS + 1];   // prefix of tiles (x parties) per job
    int64_t kps[SEG_MAX_JOBS];              // K slice per cluster rank, multiple of BK
    int tiles_n[SEG_MAX_JOBS], tiles_m[SEG_MAX_JOBS];
    int njobs, ks;
};

// epilogue adapter for cl_finish
template <typename T>
struct SegEpi {
    const SegArgs<T> *a;
    int64_t M, N;
    __device__ __forceinline__ T zload(int p, int64_t m, int64_t n) const { return a->Z[p][m * N + n]; }
    __device__ __forceinline__ void put(int p, int64_t m, int64_t n, T acc, T z) const {
        a->C[p][m * N + n] = trunc_share<T>(acc + z, a->party[p], a->trunc);
    }
};

struct SegCfg {
    static constexpr int BM = 32, BN = 32, BK = 16, NT = 256, TM = 2, TN = 2, STAGES = 4;
    static constexpr int TX = BN / TN;
    static constexpr int A_WORDS = BM * BK, B_WORDS = BK * BN;
    static constexpr int SMEM_WORDS = STAGES * (A_WORDS + B_WORDS);
    static_assert(SMEM_WORDS >= BM * BN, "reduction buffer must fit");
};

// one ring element (4 or 8 bytes) global -> shared, zero-filled when !valid
template <int BYTES>
__device__ __forceinline__ void cp_async_elem(void *smem, const void *gmem, bool valid) {
    const uint32_t s = (uint32_t)__cvta_generic_to_shared(smem);
    const int n = valid ? BYTES : 0;
    asm volatile("cp.async.ca.shared.global [%0], [%1], %2, %3;" ::"r"(s), "l"(gmem), "n"(BYTES), "r"(n) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

// grid (total tiles, 1, ks), cluster (1, 1, ks)
template <typename T>
__global__ void __launch_bounds__(SegCfg::NT) seg_gemm_kernel(const __grid_constant__ SegGroup<T> g) {
    using C = SegCfg;
    __shared__ __align__(16) T smem[C::SMEM_WORDS];
    T *As = smem, *Bs = smem + C::STAGES * C::A_WORDS;   // As[s][mm][kk], Bs[s][kb][nn]
    const int64_t t = blockIdx.x;
    int jb = 0;
#pragma unroll
    for (int q = 1; q < SEG_MAX_JOBS; ++q)
        if (q < g.njobs && t >= g.tile_begin[q]) jb = q;
    const SegArgs<T> &a = g.j[jb];
    const int64_t tt = t - g.tile_begin[jb];
    const int64_t per_party = (int64_t)g.tiles_m[jb] * g.tiles_n[jb];
    const int p = (int)(tt / per_party);
    const int64_t tp = tt - p * per_party;
    const int64_t m0 = (tp / g.tiles_n[jb]) * C::BM, n0 = (tp % g.tiles_n[jb]) * C::BN;
    const int ks = g.ks, split = blockIdx.z;
    const int64_t K = a.K, Kext = 2 * K;
    const int64_t kbeg = (int64_t)split * g.kps[jb], kend = min(Kext, kbeg + g.kps[jb]);
    const int nch = kend > kbeg ? (int)((kend - kbeg + C::BK - 1) / C::BK) : 0;
    const int tid = threadIdx.x;
    const T *Xp = a.X[p], *Vp = a.V[p];
    pdl_trigger();
    // the epilogue's Z_p words are dealer material, complete before any PDL predecessor started
    // (dealer kernels never trigger early): load them while the predecessor finishes
    SegEpi<T> epi{&a, a.M, a.N};
    T zpre[cl_zpre_n<C>()];
    cl_zload<T, SegEpi<T>, C>(epi, p, m0, n0, ks, ks > 1 ? (int)cooperative_groups::this_cluster().block_rank() : 0,
                              zpre);
    pdl_wait();   // operands come from the predecessor
    auto issue = [&](int c) {
        const int st = c % C::STAGES;
        const int64_t k0 = kbeg + (int64_t)c * C::BK;
#pragma unroll
        for (int u = 0; u < C::A_WORDS / C::NT; ++u) {
            const int idx = tid + u * C::NT, mm = idx / C::BK, kk = idx % C::BK;
            const int64_t m = m0 + mm, k = k0 + kk;
            const bool ok = m < a.M && k < kend;
            const int64_t mc = m < a.M ? m : a.M - 1, kc = k < kend ? k : kend - 1;
            const T *src = kc < K ? Xp + mc * K + kc : a.E + mc * K + (kc - K);
            cp_async_elem<sizeof(T)>(As + st * C::A_WORDS + idx, src, ok);
        }
#pragma unroll
        for (int u = 0; u < C::B_WORDS / C::NT; ++u) {
            const int idx = tid + u * C::NT, kb = idx / C::BN, nn = idx % C::BN;
            const int64_t k = k0 + kb, n = n0 + nn;
            const bool ok = n < a.N && k < kend;
            const int64_t kc = k < kend ? k : kend - 1, nc = n < a.N ? n : a.N - 1;
            const T *src = kc < K ? a.F + kc * a.N + nc : Vp + (kc - K) * a.N + nc;
            cp_async_elem<sizeof(T)>(Bs + st * C::B_WORDS + idx, src, ok);
        }
    };
#pragma unroll
    for (int c = 0; c < C::STAGES - 1; ++c) {
        if (c < nch) issue(c);
        cp_async_commit();
    }
    const int tx = tid % C::TX, ty = tid / C::TX;
    RingAcc<T> r[C::TM][C::TN];
#pragma unroll
    for (int i = 0; i < C::TM; ++i)
#pragma unroll
        for (int j = 0; j < C::TN; ++j) r[i][j].zero();
    for (int c = 0; c < nch; ++c) {
        cp_async_wait<C::STAGES - 2>();
        __syncthreads();
        if (c + C::STAGES - 1 < nch) issue(c + C::STAGES - 1);
        cp_async_commit();
        const T *as = As + (c % C::STAGES) * C::A_WORDS, *bs = Bs + (c % C::STAGES) * C::B_WORDS;
#pragma unroll
        for (int kk = 0; kk < C::BK; ++kk) {
            T av[C::TM], bv[C::TN];
#pragma unroll
            for (int i = 0; i < C::TM; ++i) av[i] = as[(ty + i * (C::BM / C::TM)) * C::BK + kk];
#pragma unroll
            for (int j = 0; j < C::TN; ++j) bv[j] = bs[kk * C::BN + tx + j * C::TX];
#pragma unroll
            for (int i = 0; i < C::TM; ++i)
#pragma unroll
                for (int j = 0; j < C::TN; ++j) r[i][j].mac(av[i], bv[j]);
        }
    }
    cp_async_wait<0>();
    T acc[C::TM][C::TN];
#pragma unroll
    for (int i = 0; i < C::TM; ++i)
#pragma unroll
        for (int j = 0; j < C::TN; ++j) acc[i][j] = r[i][j].value();
    cl_finish<T, SegEpi<T>, C>(epi, p, m0, n0, ks, smem, acc, zpre);
}

// tcgen05 form of the same group (gemm_tcseg.cu; l = 64, sm_100, K' <= 16384 per product).
// PSML_SEG=simt keeps the CUDA-core kernel below.
bool tc_seg_enabled();
bool tc_seg_forced();   // PSML_SEG=tc: every eligible group on tcgen05 (tests)
bool pdl_enabled();     // PSML_PDL=0 disables programmatic dependent launch
// segs = 2: Beaver products [X_p | E] . [F ; V_p]; 1: plain X . F.  fill: the grid's K split stops at
// 2/fill of the SMs (2 inside the training step, whose dealer branch runs beside it; 0 stand-alone:
// one wave of one-CTA-per-SM clusters).
#ifndef PSML_TCSEG_FILL
#define PSML_TCSEG_FILL 2
#endif
psml_status tc_seg_group(const SegArgs<uint64_t> *jobs, int njobs, cudaStream_t stream, int sm_count, int segs = 2,
                         int fill = PSML_TCSEG_FILL);
// Stand-alone products on the in-kernel limb-split kernel (psml_options.tc_small): plain C = A . B
// and the co-resident Beaver product (one mask + open pass, then Eq. 8); l = 64 needs K' <= 16384.
bool tc_seg_small(int l, int64_t M, int64_t Kext, int64_t N, int nparty, int sm_count);
template <typename T>
psml_status tc_seg_plain(const T *A, const T *B, int64_t M, int64_t K, int64_t N, T *C, cudaStream_t s, int sm_count);
template <typename T>
size_t tc_seg_beaver_ws_bytes(int64_t M, int64_t K, int64_t N);
template <typename T>
psml_status tc_seg_beaver(const T *const A[2], const T *const B[2], const T *const U[2], const T *const V[2],
                          const T *const Z[2], int64_t M, int64_t K, int64_t N, int flags, int trunc, T *const C[2],
                          void *ws, size_t ws_bytes, cudaStream_t s, int sm_count);


// Launch 1..SEG_MAX_JOBS products as one grid; the cluster split ks is chosen for the group.
template <typename T>
psml_status launch_seg_group(const SegArgs<T> *jobs, int njobs, cudaStream_t stream, int sm_count) {
    using C = SegCfg;
    if (njobs < 1 || njobs > SEG_MAX_JOBS) return fail(PSML_ERR_INVALID, "seg group: 1..4 jobs");
    if constexpr (sizeof(T) == 8) {
        // tcgen05 once the group has >= 2^25 ring MACs (measured on B200, tools/gpu53-55.sh: the
        // 128 x 1568 x 128 and 784 x 256 x 128 products of the MLP run 1.4x faster on tcgen05;
        // the smaller ones are bound by its fixed ~7 us prologue + DSMEM split-K reduction)
        bool ok = tc_seg_enabled();
        double macs = 0;
        for (int q = 0; q < njobs && ok; ++q) {
            ok = 2 * jobs[q].K <= 16384;
            macs += (double)jobs[q].M * jobs[q].N * 2 * jobs[q].K * jobs[q].nparty;
        }
        if (ok && (macs >= (double)(1 << 25) || tc_seg_forced()))
            return tc_seg_group(reinterpret_cast<const SegArgs<uint64_t> *>(jobs), njobs, stream, sm_count);
    }
    SegGroup<T> g{};
    int64_t tiles = 0, kmax = 0;
    double work = 0;
    for (int q = 0; q < njobs; ++q) {
        g.j[q] = jobs[q];
        g.tiles_m[q] = (int)((jobs[q].M + C::BM - 1) / C::BM);
        g.tiles_n[q] = (int)((jobs[q].N + C::BN - 1) / C::BN);
        g.tile_begin[q] = tiles;
        tiles += (int64_t)g.tiles_m[q] * g.tiles_n[q] * jobs[q].nparty;
        kmax = std::max<int64_t>(kmax, 2 * jobs[q].K);
        work += (double)jobs[q].M * jobs[q].N * 2 * jobs[q].K * jobs[q].nparty;
    }
    g.tile_begin[njobs] = tiles;
    g.njobs = njobs;
    g.ks = cl_splits(tiles, kmax, sm_count);
    for (int q = 0; q < njobs; ++q) {
        const int64_t kps = (2 * jobs[q].K + g.ks - 1) / g.ks;
        g.kps[q] = ((kps + C::BK - 1) / C::BK) * C::BK;
    }
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)tiles, 1, (unsigned)g.ks);
    cfg.blockDim = dim3(C::NT);
    cfg.stream = stream;
    cudaLaunchAttribute attr[2];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = 1; attr[0].val.clusterDim.y = 1; attr[0].val.clusterDim.z = (unsigned)g.ks;
    attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[1].val.programmaticStreamSerializationAllowed = pdl_enabled() ? 1 : 0;
    cfg.attrs = attr;
    cfg.numAttrs = 2;
    ProfScope prof(PROF_GEMM, stream, work);
    PSML_CUDA_TRY(cudaLaunchKernelEx(&cfg, seg_gemm_kernel<T>, g));
    return PSML_OK;
}

template <typename T>
psml_status launch_seg_gemm(SegArgs<T> a, int nparty, cudaStream_t stream, int sm_count) {
    a.nparty = nparty;
    return launch_seg_group<T>(&a, 1, stream, sm_count);
}

template <typename T>
psml_status launch_open(const OpenJobs<T> &jobs, cudaStream_t s) {
    int64_t maxt = 0;
    for (int q = 0; q < 2; ++q)
        maxt = std::max(maxt, ((jobs.j[q].rows + 31) / 32) * ((jobs.j[q].cols + 31) / 32));
    ProfScope prof(PROF_MASK, s, 0.0);
    open_kernel<T><<<dim3((unsigned)std::min<int64_t>(maxt, 148 * 8), 1, 2), dim3(32, 8), 0, s>>>(jobs);
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

// The product is small enough for the cluster kernels (and not a GEMV).
inline bool seg_eligible(int64_t M, int64_t K, int64_t N, int nparty) {
    (void)K;
    return !(N <= 2 && M * nparty <= 4096) && M * N * nparty <= ((int64_t)1 << 19);
}

}  // namespace psml
