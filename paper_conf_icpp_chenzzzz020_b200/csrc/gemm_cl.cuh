// gemm_cl.cuh -- latency-oriented CUDA-core ring GEMM for the small products of the paper's
// training workloads (MLP 128 x 784 x 128 ... 128 x 128 x 10, Sec. 7.1), included by
// gemm_simt.cuh.
//
// One CTA = NT threads = one BM x BN output tile of one party over one K slice; each thread holds
// TM x TN accumulators.  For l = 64 each accumulator is split into a 64-bit sum of lo.lo products
// (IMAD.WIDE.U32 with accumulate) and a 32-bit sum of the cross terms lo.hi + hi.lo, combined once
// at the end: 3 IMADs per ring MAC instead of 5 (exact: a.b mod 2^64 = lo.lo + (cross mod 2^32) << 32).
// K is split over the KS CTAs of a thread-block cluster (1, 1, KS); the partial tiles are summed
// through distributed shared memory (each CTA reduces 1/KS of the tile and runs the epilogue on
// it), so split-K needs no atomics, no workspace and no second launch.  Ring addition is exact,
// so the result is independent of KS (bit-identical, tested).
#pragma once
#include <cooperative_groups.h>

#include "common.cuh"

namespace psml {

template <int BM_, int BN_, int NT_, int TM_, int TN_, int BK_ = 32>
struct ClCfg {
    static constexpr int BM = BM_, BN = BN_, BK = BK_, NT = NT_, TM = TM_, TN = TN_;
    static constexpr int AP = BM + 1, BP = BN + 1;   // padded rows (64-bit banks)
    static constexpr int SMEM_WORDS = 2 * BK * AP + 2 * BK * BP;
    static constexpr int A_PER = BM * BK / NT, B_PER = BK * BN / NT;
    static constexpr int TX = BN / TN;   // threads along n
    static_assert((BM / TM) * (BN / TN) == NT, "thread tile mismatch");
    static_assert(A_PER * NT == BM * BK && B_PER * NT == BK * BN, "load mismatch");
    static_assert(SMEM_WORDS >= BM * BN, "reduction buffer must fit");
};
using ClDefault = ClCfg<32, 32, 256, 2, 2, 16>;   // measured best on the MLP shapes (tools/micro)
// the dealer's Z = U V products run beside the online phase: 4 x 4 outputs per thread halve the
// shared-memory words per ring MAC (PSML_DEAL_TILE=64)
using ClDealer = ClCfg<64, 64, 256, 4, 4, 16>;

// RingAcc (split-accumulator ring MAC) lives in gemm_simt.cuh, which includes this file.

template <typename T, class Ops, class C>
__device__ __forceinline__ void cl_tile(const Ops &ops, int p, int64_t m0, int64_t n0, int64_t kbeg, int64_t kend,
                                        T *smem, T acc[C::TM][C::TN]) {
    constexpr int BM = C::BM, BN = C::BN, BK = C::BK, NT = C::NT, AP = C::AP, BP = C::BP;
    T(*As)[BK][AP] = reinterpret_cast<T(*)[BK][AP]>(smem);
    T(*Bs)[BK][BP] = reinterpret_cast<T(*)[BK][BP]>(smem + 2 * BK * AP);
    const int tid = threadIdx.x;
    const int tx = tid % C::TX, ty = tid / C::TX;   // outputs rows ty + i*(BM/TM), cols tx + j*TX
    const bool ak = ops_a_kmajor(ops, 0), bn = ops_b_nmajor(ops, 0);
    T ra[C::A_PER], rb[C::B_PER];
    auto load = [&](int64_t k0) {
#pragma unroll
        for (int t = 0; t < C::A_PER; ++t) {
            const int idx = tid + t * NT;
            const int mm = ak ? (idx / BK) : (idx % BM), kk = ak ? (idx % BK) : (idx / BM);
            const int64_t m = m0 + mm, k = k0 + kk;
            const T va = ops.a(p, m < ops.M ? m : ops.M - 1, k < kend ? k : kend - 1);   // clamped: no branch
            ra[t] = (m < ops.M && k < kend) ? va : (T)0;
        }
#pragma unroll
        for (int t = 0; t < C::B_PER; ++t) {
            const int idx = tid + t * NT;
            const int kb = bn ? (idx / BN) : (idx % BK), nn = bn ? (idx % BN) : (idx / BK);
            const int64_t k2 = k0 + kb, n = n0 + nn;
            const T vb = ops.b(p, k2 < kend ? k2 : kend - 1, n < ops.N ? n : ops.N - 1);
            rb[t] = (n < ops.N && k2 < kend) ? vb : (T)0;
        }
    };
    auto stash = [&](int buf) {
#pragma unroll
        for (int t = 0; t < C::A_PER; ++t) {
            const int idx = tid + t * NT;
            const int mm = ak ? (idx / BK) : (idx % BM), kk = ak ? (idx % BK) : (idx / BM);
            As[buf][kk][mm] = ra[t];
        }
#pragma unroll
        for (int t = 0; t < C::B_PER; ++t) {
            const int idx = tid + t * NT;
            const int kb = bn ? (idx / BN) : (idx % BK), nn = bn ? (idx % BN) : (idx / BK);
            Bs[buf][kb][nn] = rb[t];
        }
    };
    RingAcc<T> r[C::TM][C::TN];
#pragma unroll
    for (int i = 0; i < C::TM; ++i)
#pragma unroll
        for (int j = 0; j < C::TN; ++j) r[i][j].zero();
    int buf = 0;
    if (kbeg < kend) { load(kbeg); stash(0); }
    __syncthreads();
    for (int64_t k0 = kbeg; k0 < kend; k0 += BK) {
        const bool more = k0 + BK < kend;
        if (more) load(k0 + BK);
#pragma unroll 8
        for (int kk = 0; kk < BK; ++kk) {
            T a[C::TM], b[C::TN];
#pragma unroll
            for (int i = 0; i < C::TM; ++i) a[i] = As[buf][kk][ty + i * (BM / C::TM)];
#pragma unroll
            for (int j = 0; j < C::TN; ++j) b[j] = Bs[buf][kk][tx + j * C::TX];
#pragma unroll
            for (int i = 0; i < C::TM; ++i)
#pragma unroll
                for (int j = 0; j < C::TN; ++j) r[i][j].mac(a[i], b[j]);
        }
        if (more) {
            stash(buf ^ 1);
            __syncthreads();
            buf ^= 1;
        }
    }
#pragma unroll
    for (int i = 0; i < C::TM; ++i)
#pragma unroll
        for (int j = 0; j < C::TN; ++j) acc[i][j] = r[i][j].value();
}

// Store (KS == 1) or cluster-reduce + store one tile.  `red` = this CTA's smem (>= BM x BN words).
// Epilogue Z words of this thread (the order cl_finish consumes them), for kernels that load them
// ahead of time (before griddepcontrol.wait): ks == 1 -> TM x TN outputs of the thread; ks > 1 ->
// the thread's elements of this CTA's 1/ks slice of the reduced tile.
template <class C> constexpr int cl_zpre_n() {
    return C::TM * C::TN > (C::BM * C::BN + 2 * C::NT - 1) / (2 * C::NT) ? C::TM * C::TN
                                                                       : (C::BM * C::BN + 2 * C::NT - 1) / (2 * C::NT);
}
template <typename T, class Ops, class C>
__device__ __forceinline__ void cl_zload(const Ops &ops, int p, int64_t m0, int64_t n0, int ks, int rank,
                                         T z[cl_zpre_n<C>()]) {
    constexpr int BM = C::BM, BN = C::BN, NT = C::NT;
    const int tid = threadIdx.x, tx = tid % C::TX, ty = tid / C::TX;
    if (ks == 1) {
#pragma unroll
        for (int i = 0; i < C::TM; ++i)
#pragma unroll
            for (int j = 0; j < C::TN; ++j) {
                const int64_t m = m0 + ty + i * (BM / C::TM), n = n0 + tx + j * C::TX;
                z[i * C::TN + j] = ops.zload(p, m < ops.M ? m : ops.M - 1, n < ops.N ? n : ops.N - 1);
            }
        return;
    }
    constexpr int MAXC = (BM * BN + 2 * NT - 1) / (2 * NT);
    const int per = (BM * BN) / ks;
#pragma unroll
    for (int u = 0; u < MAXC; ++u) {
        z[u] = 0;
        if (tid + u * NT < per) {
            const int e = rank * per + tid + u * NT;
            const int64_t m = m0 + e / BN, n = n0 + e % BN;
            z[u] = ops.zload(p, m < ops.M ? m : ops.M - 1, n < ops.N ? n : ops.N - 1);
        }
    }
}

template <typename T, class Ops, class C>
__device__ __forceinline__ void cl_finish(const Ops &ops, int p, int64_t m0, int64_t n0, int ks, T *red,
                                          T acc[C::TM][C::TN], const T *zpre = nullptr) {
    constexpr int BM = C::BM, BN = C::BN, NT = C::NT;
    const int tid = threadIdx.x, tx = tid % C::TX, ty = tid / C::TX;
    if (ks == 1) {   // epilogue operands first (clamped, unconditional), then the stores
        T z[C::TM][C::TN];
#pragma unroll
        for (int i = 0; i < C::TM; ++i)
#pragma unroll
            for (int j = 0; j < C::TN; ++j) {
                const int64_t m = m0 + ty + i * (BM / C::TM), n = n0 + tx + j * C::TX;
                z[i][j] = zpre ? zpre[i * C::TN + j] : ops.zload(p, m < ops.M ? m : ops.M - 1, n < ops.N ? n : ops.N - 1);
            }
#pragma unroll
        for (int i = 0; i < C::TM; ++i)
#pragma unroll
            for (int j = 0; j < C::TN; ++j) {
                const int64_t m = m0 + ty + i * (BM / C::TM), n = n0 + tx + j * C::TX;
                if (m < ops.M && n < ops.N) ops.put(p, m, n, acc[i][j], z[i][j]);
            }
        return;
    }
    namespace cg = cooperative_groups;
    cg::cluster_group cluster = cg::this_cluster();
    const int rank = (int)cluster.block_rank();
    constexpr int MAXC = (BM * BN + 2 * NT - 1) / (2 * NT);   // ks >= 2
    const int per = (BM * BN) / ks;                              // ks divides BM * BN (power of two)
    T sum[MAXC], zz[MAXC];
    // this CTA's epilogue Z words first: their load latency overlaps the partial-tile exchange
#pragma unroll
    for (int u = 0; u < MAXC; ++u) {
        zz[u] = 0;
        if (tid + u * NT < per) {
            const int e = rank * per + tid + u * NT;
            const int64_t m = m0 + e / BN, n = n0 + e % BN;
            zz[u] = zpre ? zpre[u] : ops.zload(p, m < ops.M ? m : ops.M - 1, n < ops.N ? n : ops.N - 1);
        }
    }
    __syncthreads();   // all warps done with the operand tiles that `red` overlays
#pragma unroll
    for (int i = 0; i < C::TM; ++i)
#pragma unroll
        for (int j = 0; j < C::TN; ++j) red[(ty + i * (BM / C::TM)) * BN + tx + j * C::TX] = acc[i][j];
    cluster.sync();
#pragma unroll
    for (int u = 0; u < MAXC; ++u) {
        sum[u] = 0;
        if (tid + u * NT < per) {
            const int e = rank * per + tid + u * NT;
            T part[8];
#pragma unroll
            for (int q = 0; q < 8; ++q) part[q] = q < ks ? cluster.map_shared_rank(red, q)[e] : (T)0;
#pragma unroll
            for (int q = 0; q < 8; ++q) sum[u] += part[q];
        }
    }
#pragma unroll
    for (int u = 0; u < MAXC; ++u) {
        if (tid + u * NT < per) {
            const int e = rank * per + tid + u * NT;
            const int64_t m = m0 + e / BN, n = n0 + e % BN;
            if (m < ops.M && n < ops.N) ops.put(p, m, n, sum[u], zz[u]);
        }
    }
    // peers' shared memory stays alive until every CTA has read it (the reads completed: their
    // values were summed above), so no memory ordering is needed here
    asm volatile("barrier.cluster.arrive.relaxed.aligned;\nbarrier.cluster.wait.aligned;" ::: "memory");
}

// One product: grid (ceil(N/BN), ceil(M/BM), nparty * ks), cluster (1, 1, ks).
template <typename T, class Ops, class C = ClDefault>
__global__ void __launch_bounds__(C::NT) ring_gemm_cl(Ops ops, int ks, int64_t k_per_split) {
    __shared__ __align__(16) T smem[C::SMEM_WORDS];
    const int p = blockIdx.z / ks, split = blockIdx.z % ks;
    const int64_t m0 = (int64_t)blockIdx.y * C::BM, n0 = (int64_t)blockIdx.x * C::BN;
    const int64_t kbeg = (int64_t)split * k_per_split, kend = min(ops.Kext, kbeg + k_per_split);
    T acc[C::TM][C::TN];
    cl_tile<T, Ops, C>(ops, p, m0, n0, kbeg, kend, smem, acc);
    cl_finish<T, Ops, C>(ops, p, m0, n0, ks, smem, acc);
}

// Several independent single-party products in one launch (the dealer's Z = U V of one step):
// grid (total tiles, 1, ks), cluster (1, 1, ks); job found from the tile index.
template <class Ops>
struct ClJob {
    Ops ops;
    int64_t tile_begin, k_per_split;
    int tiles_n;
};

template <typename T, class Ops, class C = ClDefault>
__global__ void __launch_bounds__(C::NT) ring_gemm_cl_grouped(const ClJob<Ops> *__restrict__ jobs, int njobs, int ks) {
    __shared__ __align__(16) T smem[C::SMEM_WORDS];
    const int64_t t = blockIdx.x;
    int lo = 0, hi = njobs - 1;
    while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (jobs[mid].tile_begin <= t) lo = mid; else hi = mid - 1;
    }
    const Ops ops = jobs[lo].ops;
    const int64_t tt = t - jobs[lo].tile_begin, kps = jobs[lo].k_per_split;
    const int64_t m0 = (tt / jobs[lo].tiles_n) * C::BM, n0 = (tt % jobs[lo].tiles_n) * C::BN;
    const int split = blockIdx.z;
    const int64_t kbeg = (int64_t)split * kps, kend = min(ops.Kext, kbeg + kps);
    T acc[C::TM][C::TN];
    cl_tile<T, Ops, C>(ops, 0, m0, n0, kbeg, kend, smem, acc);
    cl_finish<T, Ops, C>(ops, 0, m0, n0, ks, smem, acc);
}

// K split for a product with `tiles` output tiles: power of two <= 8 keeping <= `waves` CTAs per
// SM, each slice >= `min_chunks` chunks deep.
inline int cl_splits(int64_t tiles, int64_t Kext, int sm_count, int waves = 8, int min_chunks = 1) {
    int ks = 1;
    while (ks < 8 && tiles * ks * 2 <= (int64_t)sm_count * waves && Kext / (ks * 2) >= min_chunks * 16) ks *= 2;
    return ks;
}

template <typename T, class Ops, class C = ClDefault>
psml_status launch_ring_gemm_cl(const Ops &ops, cudaStream_t stream, int sm_count, int ks = 0) {
    const int64_t tiles = ((ops.M + C::BM - 1) / C::BM) * ((ops.N + C::BN - 1) / C::BN) * Ops::nparty;
    if (ks <= 0) ks = cl_splits(tiles, ops.Kext, sm_count);
    int64_t kps = (ops.Kext + ks - 1) / ks;
    kps = ((kps + C::BK - 1) / C::BK) * C::BK;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)((ops.N + C::BN - 1) / C::BN), (unsigned)((ops.M + C::BM - 1) / C::BM),
                       (unsigned)(Ops::nparty * ks));
    cfg.blockDim = dim3(C::NT);
    cfg.stream = stream;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = 1; attr[0].val.clusterDim.y = 1; attr[0].val.clusterDim.z = (unsigned)ks;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    PSML_CUDA_TRY(cudaLaunchKernelEx(&cfg, ring_gemm_cl<T, Ops, C>, ops, ks, kps));
    return PSML_OK;
}

}  // namespace psml
