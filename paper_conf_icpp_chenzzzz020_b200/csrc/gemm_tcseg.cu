// gemm_tcseg.cu -- the opened Beaver product of the training step (Eq. 8:
// C_p = [X_p | E] . [F ; V_p] + Z_p, then SecureML truncation) on the tcgen05 tensor cores, for
// the small products of the paper's workloads (MLP 128 x 784 x 128 ... 784 x 128 x 128).
//
// Same exact limb decomposition as gemm_tc.cu (8-bit limbs, the 36 limb pairs p + q < 8 of Z_2^64
// as tcgen05.mma.kind::i8 into 8 per-shift s32 TMEM accumulators S_s, result sum_s S_s 2^{8s}),
// but built for products whose whole operand set is a few MB: there is NO separate limb-split
// pass through HBM.  The CTA's 8 warps load the uint64 operand words straight from the producers'
// outputs (L2-resident), split them into limb bytes in registers (a 4 x 4 byte transpose per
// 4 words: 2 PRMT per limb word) and store them into shared memory already in the UMMA K-major
// no-swizzle canonical layout; one thread issues the 36 MMAs of the 128 x 64 x 32 block while the
// warps split the next block (3-stage ring; the commit of a stage's MMAs frees it).
// K is split over the ks CTAs of a (1, 1, ks) thread-block cluster: each CTA turns its
// accumulators into uint64 partials (exact mod 2^64, K' per CTA <= 2^14 keeps S_0..S_3 exact),
// the partial tiles are summed through distributed shared memory, and each CTA runs the epilogue
// (+ Z_p, truncation, store) on 1/ks of the tile.  Ring addition is exact, so the result is
// bit-identical to the CUDA-core seg_gemm_kernel (tested).
#ifndef PSML_TCSEG_FILL
#define PSML_TCSEG_FILL 2
#endif
#include <cooperative_groups.h>

#include "engine.h"

namespace psml {
namespace tcseg {

constexpr int BM = 128, BN = 64, BK = 32, NT = 256, STAGES = 2, L = 8;
constexpr int NTH = NT + 32;   // NT producer threads (loads, limb split, epilogue) + the MMA warp
constexpr int A_TILE = BM * BK;                     // bytes per limb plane of one A block
constexpr int B_TILE = BN * BK;                     // bytes per limb plane of one B block
constexpr int STAGE_BYTES = L * (A_TILE + B_TILE);  // 48 KB of limb planes per K block
constexpr int RED_PITCH = BN + 1;                   // u64 words per row of the reduction tile
// raw uint64 operand words of one K block, landed by cp.async two blocks ahead of their split
constexpr int RAW_STAGES = 2, RAW_A_PITCH = 34;     // A rows padded to 272 B (16-B aligned)
constexpr int RAW_A_BYTES = BM * RAW_A_PITCH * 8, RAW_B_BYTES = BK * BN * 8;
constexpr int RAW_STAGE_BYTES = RAW_A_BYTES + RAW_B_BYTES;
constexpr int RAW_OFF = STAGES * STAGE_BYTES;
constexpr int PIPE_BYTES = RAW_OFF + RAW_STAGES * RAW_STAGE_BYTES;
static_assert(BM * RED_PITCH * 8 <= PIPE_BYTES, "reduction tile must fit the pipeline region");
constexpr size_t SMEM_BYTES = PIPE_BYTES + 8 * (2 * STAGES + 2) + 16;   // > 114 KB: one CTA per SM
constexpr int MAX_KS = 16;

struct Group {
    SegArgs<uint64_t> j[SEG_MAX_JOBS];
    int64_t tile_begin[SEG_MAX_JOBS + 1];
    int tiles_n[SEG_MAX_JOBS], tiles_m[SEG_MAX_JOBS];
    int kb_per_split[SEG_MAX_JOBS];
    int njobs, ks;
};

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
    asm volatile(
        "{\n"
        ".reg .pred P1;\n"
        "TCSEG_WAIT:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
        "@P1 bra TCSEG_DONE;\n"
        "bra TCSEG_WAIT;\n"
        "TCSEG_DONE:\n"
        "}\n" ::"r"(bar),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void mma_i8(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
    asm volatile(
        "{\n"
        ".reg .pred p;\n"
        "setp.ne.b32 p, %4, 0;\n"
        "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n"
        "}\n" ::"r"(d),
        "l"(a), "l"(b), "r"(idesc), "r"(acc)
        : "memory");
}
__device__ __forceinline__ void commit(uint32_t bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t r[16]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, "
        "%15}, [%16];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]),
          "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
        : "r"(taddr));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}
// four 32x32b.x16 TMEM loads and their wait in ONE asm statement (the registers cannot be
// consumed before the wait)
__device__ __forceinline__ void tmem_ld16x4(uint32_t t0, uint32_t t1, uint32_t t2, uint32_t t3, uint32_t r[64]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, %15}, [%64];\n"
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31}, [%65];\n"
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%32, %33, %34, %35, %36, %37, %38, %39, %40, %41, %42, %43, %44, %45, %46, %47}, [%66];\n"
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%48, %49, %50, %51, %52, %53, %54, %55, %56, %57, %58, %59, %60, %61, %62, %63}, [%67];\n"
        "tcgen05.wait::ld.sync.aligned;\n"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31]), "=r"(r[32]), "=r"(r[33]), "=r"(r[34]), "=r"(r[35]), "=r"(r[36]), "=r"(r[37]), "=r"(r[38]), "=r"(r[39]), "=r"(r[40]), "=r"(r[41]), "=r"(r[42]), "=r"(r[43]), "=r"(r[44]), "=r"(r[45]), "=r"(r[46]), "=r"(r[47]), "=r"(r[48]), "=r"(r[49]), "=r"(r[50]), "=r"(r[51]), "=r"(r[52]), "=r"(r[53]), "=r"(r[54]), "=r"(r[55]), "=r"(r[56]), "=r"(r[57]), "=r"(r[58]), "=r"(r[59]), "=r"(r[60]), "=r"(r[61]), "=r"(r[62]), "=r"(r[63])
        : "r"(t0), "r"(t1), "r"(t2), "r"(t3)
        : "memory");
}
// UMMA shared-memory descriptor, K-major, SWIZZLE_NONE, sm_100 version bit 46.
__device__ __forceinline__ uint64_t sdesc(uint32_t addr) {
    return (uint64_t)((addr >> 4) & 0x3FFFu) | ((uint64_t)(128 >> 4) << 16) | ((uint64_t)(256 >> 4) << 32) |
           (1ull << 46);
}
// kind::i8 instruction descriptor: D s32, A/B u8, both K-major, M = BM, N = n (a multiple of 16, <= 256).
__device__ __forceinline__ uint32_t idesc_i8(int n) {
    return (2u << 4) | ((uint32_t)(n >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);
}

// 4 x 4 byte transpose: w[i] = bytes (b0..b3) of word i -> o[p] = (w0.bp, w1.bp, w2.bp, w3.bp)
__device__ __forceinline__ void bt4(uint32_t w0, uint32_t w1, uint32_t w2, uint32_t w3, uint32_t o[4]) {
    const uint32_t t0 = __byte_perm(w0, w1, 0x5140), t1 = __byte_perm(w0, w1, 0x7362);
    const uint32_t t2 = __byte_perm(w2, w3, 0x5140), t3 = __byte_perm(w2, w3, 0x7362);
    o[0] = __byte_perm(t0, t2, 0x5410);
    o[1] = __byte_perm(t0, t2, 0x7632);
    o[2] = __byte_perm(t1, t3, 0x5410);
    o[3] = __byte_perm(t1, t3, 0x7632);
}
// limb words of 4 consecutive ring elements: out[p] = bytes p of v0..v3 (p = 0..7)
__device__ __forceinline__ void limbs4(const uint64_t *v, uint32_t out[8]) {
    bt4((uint32_t)v[0], (uint32_t)v[1], (uint32_t)v[2], (uint32_t)v[3], out);
    bt4((uint32_t)(v[0] >> 32), (uint32_t)(v[1] >> 32), (uint32_t)(v[2] >> 32), (uint32_t)(v[3] >> 32), out + 4);
}

__device__ __forceinline__ uint64_t ldg(const uint64_t *p) { return __ldg((const unsigned long long *)p); }
__device__ __forceinline__ void cp_async16(void *dst, const void *src, bool ok) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(smem_u32(dst)), "l"(src), "r"(ok ? 16 : 0)
                 : "memory");
}
__device__ __forceinline__ void cp_async8(void *dst, const void *src, bool ok) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;" ::"r"(smem_u32(dst)), "l"(src), "r"(ok ? 8 : 0)
                 : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait1() { asm volatile("cp.async.wait_group 1;" ::: "memory"); }

constexpr int ZPF = 8;   // epilogue Z words prefetched per thread (ks >= 4)

// Epilogue of this CTA's reduced slice (rows [rank R, (rank + 1) R) of the tile, R = BM / KS):
// thread tid owns elements e = rank * PER + tid + NT * i (i < NEL); + Z_p, truncation, store.
template <int KS>
__device__ __forceinline__ void slice_store(const SegArgs<uint64_t> &a, int p, int64_t m0, int64_t n0, int rank,
                                            const uint64_t *red, const uint64_t zpre[ZPF]) {
    constexpr int PER = BM * BN / KS, NEL = PER / NT;
    const int tid = threadIdx.x, party = a.party[p];
#pragma unroll
    for (int i = 0; i < NEL; ++i) {
        const int e = rank * PER + tid + NT * i;
        const int r = e / BN, c = e % BN;
        const int64_t m = m0 + r, n = n0 + c;
        const int64_t off = (m < a.M ? m : a.M - 1) * a.N + (n < a.N ? n : a.N - 1);
        const uint64_t z = NEL <= ZPF ? zpre[i < ZPF ? i : 0] : ldg(a.Z[p] + off);
        const uint64_t sum = red[r * RED_PITCH + c];
        if (m < a.M && n < a.N) a.C[p][off] = trunc_share<uint64_t>(sum + z, party, a.trunc);
    }
}

// The same epilogue, summing the slice's rows straight out of every cluster CTA's partial tile
// (ld.shared::cluster: distributed shared memory reads, KS loads per element in flight).
template <int KS>
__device__ __forceinline__ void slice_sum_store(const SegArgs<uint64_t> &a, int p, int64_t m0, int64_t n0, int rank,
                                                uint32_t red_u32, const uint64_t zpre[ZPF]) {
    constexpr int PER = BM * BN / KS, NEL = PER / NT;
    const int tid = threadIdx.x, party = a.party[p];
    uint32_t peer[KS];
#pragma unroll
    for (int q = 0; q < KS; ++q) asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(peer[q]) : "r"(red_u32), "r"(q));
#pragma unroll
    for (int i = 0; i < NEL; ++i) {
        const int e = rank * PER + tid + NT * i;
        const int r = e / BN, c = e % BN;
        const uint32_t off = (uint32_t)(r * RED_PITCH + c) * 8;
        uint64_t part[KS];
#pragma unroll
        for (int q = 0; q < KS; ++q) asm volatile("ld.shared::cluster.u64 %0, [%1];" : "=l"(part[q]) : "r"(peer[q] + off));
        uint64_t sum = 0;
#pragma unroll
        for (int q = 0; q < KS; ++q) sum += part[q];
        const int64_t m = m0 + r, n = n0 + c;
        const int64_t o = (m < a.M ? m : a.M - 1) * a.N + (n < a.N ? n : a.N - 1);
        const uint64_t z = NEL <= ZPF ? zpre[i < ZPF ? i : 0] : ldg(a.Z[p] + o);
        if (m < a.M && n < a.N) a.C[p][o] = trunc_share<uint64_t>(sum + z, party, a.trunc);
    }
}

#ifndef PSML_TCSEG_RED
#define PSML_TCSEG_RED 1   // split-K reduction: 0 bulk-copy .add.u64 into the owner CTA, 1 DSMEM reads
#endif

// grid (total tiles, 1, ks), cluster (1, 1, ks), NTH threads, SMEM_BYTES dynamic shared memory.
// Warps 0-7 land the raw operand words (cp.async) and split them into limb planes; warp 8 issues
// the MMAs of each limb stage as soon as its `full` barrier completes, so the tensor core works
// on block i while the producers split block i + 1.
__global__ void __launch_bounds__(NTH, 1) tc_seg_kernel(const __grid_constant__ Group g) {
    namespace cg = cooperative_groups;
    extern __shared__ __align__(1024) uint8_t smem[];
    uint64_t *empty = (uint64_t *)(smem + PIPE_BYTES);   // limb stage free (MMAs of its block done)
    uint64_t *full = empty + STAGES;                      // limb stage written by all NT producers
    uint64_t *accum = full + STAGES;
    uint64_t *rbar = accum + 1;   // split-K reduction: peers' partial slices landed
    uint32_t *tmem_slot = (uint32_t *)(rbar + 1);
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
#ifdef TCSEG_TIMING
    uint64_t ts[9];
#define TS(i) asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(ts[i]))
    TS(0);
#else
#define TS(i)
#endif

    const int64_t t = blockIdx.x;
    int jb = 0;
#pragma unroll
    for (int q = 1; q < SEG_MAX_JOBS; ++q)
        if (q < g.njobs && t >= g.tile_begin[q]) jb = q;
    const SegArgs<uint64_t> &a = g.j[jb];
    const int64_t tt = t - g.tile_begin[jb];
    const int64_t per_party = (int64_t)g.tiles_m[jb] * g.tiles_n[jb];
    const int p = (int)(tt / per_party);
    const int64_t tp = tt - p * per_party;
    const int64_t m0 = (tp / g.tiles_n[jb]) * BM, n0 = (tp % g.tiles_n[jb]) * BN;
    const int64_t M = a.M, N = a.N, K = a.K, Kext = 2 * K;
    const int nkb = (int)((Kext + BK - 1) / BK);
    const int kb0 = (int)blockIdx.z * g.kb_per_split[jb];
    const int kb1 = min(kb0 + g.kb_per_split[jb], nkb);
    const int nblk = kb1 > kb0 ? kb1 - kb0 : 0;
    const uint64_t *Xp = a.X[p], *Ep = a.E, *Fp = a.F, *Vp = a.V[p];

    if (tid == 0) {
        for (int s = 0; s < STAGES; ++s) {
            mbar_init(smem_u32(&empty[s]), 1);
            mbar_init(smem_u32(&full[s]), NT);
        }
        mbar_init(smem_u32(accum), 1);
        mbar_init(smem_u32(rbar), 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 1) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(tmem_slot)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    fence_before();
    __syncthreads();
    fence_after();
    const uint32_t tmem = *tmem_slot;
    TS(1);
    // this CTA's epilogue elements e = rank * per + tid + NT * i (i < 32 / ks): prefetch their
    // Z_p words now (ks >= 4), so the epilogue does not wait on global memory
    uint64_t zpre[ZPF];
    {
        const int ks = g.ks, nel = (BM * BN) / ks / NT;
#pragma unroll
        for (int i = 0; i < ZPF; ++i) {
            zpre[i] = 0;
            if (nel <= ZPF && i < nel && tid < NT) {
                const int e = (int)blockIdx.z * (nel * NT) + tid + NT * i;
                const int64_t m = m0 + e / BN, n = n0 + e % BN;
                zpre[i] = ldg(a.Z[p] + (m < M ? m : M - 1) * N + (n < N ? n : N - 1));
            }
        }
    }

    // stash assignment: A unit = (row ar, 16-k half ac); B unit = (column bn, 8-k quarter bq)
    const int ar = tid >> 1, ac = tid & 1;
    const int bn = tid & 63, bq = tid >> 6;
    // cp.async of one K block's raw words into raw stage rs (zero-filled outside the operands):
    // 16-byte chunks when the X | E boundary and row starts allow it (K, N even), else 8-byte
    auto al16 = [](const void *q) { return ((uintptr_t)q & 15) == 0; };
    const bool a16 = (K % 2) == 0 && al16(Xp) && al16(Ep), b16 = (N % 2) == 0 && al16(Fp) && al16(Vp);
    auto issue = [&](int kb, int rs) {
        uint8_t *ra = smem + RAW_OFF + rs * RAW_STAGE_BYTES, *rb = ra + RAW_A_BYTES;
        const int64_t k0 = (int64_t)kb * BK;
        if (a16) {
#pragma unroll
            for (int u = 0; u < BM * BK / 2 / NT; ++u) {
                const int c = tid + NT * u, row = c >> 4, kk = (c & 15) * 2;
                const int64_t m = m0 + row, k = k0 + kk;
                const bool ok = m < M && k < Kext;
                const int64_t mc = ok ? m : 0, kc = ok ? k : 0;
                const uint64_t *src = kc < K ? Xp + mc * K + kc : Ep + mc * K + (kc - K);
                cp_async16(ra + row * RAW_A_PITCH * 8 + kk * 8, src, ok);
            }
        } else {
#pragma unroll 4
            for (int u = 0; u < BM * BK / NT; ++u) {
                const int c = tid + NT * u, row = c >> 5, kk = c & 31;
                const int64_t m = m0 + row, k = k0 + kk;
                const bool ok = m < M && k < Kext;
                const int64_t mc = ok ? m : 0, kc = ok ? k : 0;
                const uint64_t *src = kc < K ? Xp + mc * K + kc : Ep + mc * K + (kc - K);
                cp_async8(ra + row * RAW_A_PITCH * 8 + kk * 8, src, ok);
            }
        }
        if (b16) {
#pragma unroll
            for (int u = 0; u < BK * BN / 2 / NT; ++u) {
                const int c = tid + NT * u, kk = c >> 5, nn = (c & 31) * 2;
                const int64_t k = k0 + kk, n = n0 + nn;
                const bool ok = k < Kext && n < N;
                const int64_t kc = ok ? k : 0, ncl = ok ? n : 0;
                const uint64_t *src = kc < K ? Fp + kc * N + ncl : Vp + (kc - K) * N + ncl;
                cp_async16(rb + (kk * BN + nn) * 8, src, ok);
            }
        } else {
#pragma unroll 4
            for (int u = 0; u < BK * BN / NT; ++u) {
                const int c = tid + NT * u, kk = c >> 6, nn = c & 63;
                const int64_t k = k0 + kk, n = n0 + nn;
                const bool ok = k < Kext && n < N;
                const int64_t kc = ok ? k : 0, ncl = ok ? n : 0;
                const uint64_t *src = kc < K ? Fp + kc * N + ncl : Vp + (kc - K) * N + ncl;
                cp_async8(rb + (kk * BN + nn) * 8, src, ok);
            }
        }
    };
    const int a_off = (((ar >> 3) * 2 + ac) * 128) + (ar & 7) * 16;
    const int b_off = (((bn >> 3) * 2 + (bq >> 1)) * 128) + (bn & 7) * 16 + (bq & 1) * 8;
    auto stash = [&](int rs, int st) {
        const uint8_t *ra = smem + RAW_OFF + rs * RAW_STAGE_BYTES, *rb = ra + RAW_A_BYTES;
        uint8_t *sa = smem + st * STAGE_BYTES, *sb = sa + L * A_TILE;
        uint64_t va[16], vb[8];
#pragma unroll
        for (int j = 0; j < 16; j += 2) {
            const ulonglong2 v = *(const ulonglong2 *)(ra + ar * RAW_A_PITCH * 8 + (16 * ac + j) * 8);
            va[j] = v.x;
            va[j + 1] = v.y;
        }
#pragma unroll
        for (int j = 0; j < 8; ++j) vb[j] = *(const uint64_t *)(rb + ((8 * bq + j) * BN + bn) * 8);
        uint32_t w[4][8];
#pragma unroll
        for (int q = 0; q < 4; ++q) limbs4(va + 4 * q, w[q]);
#pragma unroll
        for (int l = 0; l < L; ++l)
            *(uint4 *)(sa + l * A_TILE + a_off) = make_uint4(w[0][l], w[1][l], w[2][l], w[3][l]);
        uint32_t u[2][8];
        limbs4(vb, u[0]);
        limbs4(vb + 4, u[1]);
#pragma unroll
        for (int l = 0; l < L; ++l) *(uint2 *)(sb + l * B_TILE + b_off) = make_uint2(u[0][l], u[1][l]);
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // generic writes -> tensor core
    };

    // Programmatic dependent launch: everything above (barriers, TMEM, Z prefetch -- the dealer's
    // output, complete before the predecessor kernel started) overlapped the predecessor; the
    // operands X_p / E / F it produces are read only after this wait.
    pdl_trigger();
    pdl_wait();
    if (warp < NT / 32) {   // producers
        if (nblk > 0) issue(kb0, 0);
        cp_async_commit();
        if (nblk > 1) issue(kb0 + 1, 1);
        cp_async_commit();
        TS(2);
        for (int i = 0; i < nblk; ++i) {
            const int st = i % STAGES, rs = i % RAW_STAGES;
            cp_async_wait1();                                 // this thread's chunks of block i landed
            asm volatile("bar.sync 1, %0;" ::"n"(NT) : "memory");   // ... and every producer's
            if (i >= STAGES) mbar_wait(smem_u32(&empty[st]), (uint32_t)((i / STAGES - 1) & 1));
            stash(rs, st);                                    // ends with fence.proxy.async
            asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&full[st])) : "memory");
            asm volatile("bar.sync 1, %0;" ::"n"(NT) : "memory");   // raw stage rs read by everyone
            if (i + 2 < nblk) issue(kb0 + i + 2, rs);
            cp_async_commit();
        }
    } else if (lane == 0) {   // the MMA warp: 36 limb-pair MMAs per stage into the shift accumulators
        for (int i = 0; i < nblk; ++i) {
            const int st = i % STAGES;
            mbar_wait(smem_u32(&full[st]), (uint32_t)((i / STAGES) & 1));
            fence_after();
            const uint32_t sa = smem_u32(smem + st * STAGE_BYTES), sb = sa + L * A_TILE;
            // A limb pa times B limbs 0 .. 7 - pa: the B planes lie back to back in the canonical
            // layout (plane stride = 8 row groups x SBO), so they form ONE N = 64 (8 - pa) operand
            // whose product lands in TMEM columns (pa + q) 64 = shift accumulators S_pa .. S_7 --
            // 12 MMAs of N <= 256 per K block instead of 36 of N = 64, A read from shared memory
            // 12 times instead of 36
#pragma unroll
            for (int pa = 0; pa < L; ++pa) {
                const uint64_t ad = sdesc(sa + pa * A_TILE);
#pragma unroll
                for (int q0 = 0; q0 < L - pa; q0 += 4) {
                    const int nq = (L - pa - q0) < 4 ? (L - pa - q0) : 4;
                    mma_i8(tmem + (uint32_t)((pa + q0) * BN), ad, sdesc(sb + q0 * B_TILE), idesc_i8(nq * BN),
                           (i > 0 || pa > 0) ? 1u : 0u);
                }
            }
            commit(smem_u32(&empty[st]));
        }
        commit(smem_u32(accum));
    }
    __syncwarp();
    TS(3);

    // ---- partial tile: sum_s S_s 2^{8s} (u64, exact) -> reduction buffer ----
    uint64_t *red = (uint64_t *)smem;   // the pipeline region is idle once `accum` completes
    mbar_wait(smem_u32(accum), 0);
    TS(4);
    fence_after();
    if (warp < NT / 32) {   // warps w and w + 4 share TMEM lanes 32 (w % 4) ..; each drains half the columns
        const int row = (warp & 3) * 32 + lane;
        const uint32_t lane_base = tmem + ((uint32_t)((warp & 3) * 32) << 16);
#pragma unroll 1
        for (int j0 = (warp >> 2) * (BN / 2); j0 < (warp >> 2) * (BN / 2) + BN / 2; j0 += 16) {
            uint64_t acc[16];
#pragma unroll
            for (int j = 0; j < 16; ++j) acc[j] = 0;
            if (nblk > 0) {
#pragma unroll
                for (int s0 = 0; s0 < L; s0 += 4) {   // 4 TMEM loads in flight per wait
                    uint32_t r[64];
                    tmem_ld16x4(lane_base + (uint32_t)(s0 * BN + j0), lane_base + (uint32_t)((s0 + 1) * BN + j0),
                                lane_base + (uint32_t)((s0 + 2) * BN + j0), lane_base + (uint32_t)((s0 + 3) * BN + j0), r);
#pragma unroll
                    for (int u = 0; u < 4; ++u)
#pragma unroll
                        for (int j = 0; j < 16; ++j) acc[j] += (uint64_t)r[16 * u + j] << (8 * (s0 + u));
                }
            }
#pragma unroll
            for (int j = 0; j < 16; ++j) red[row * RED_PITCH + j0 + j] = acc[j];
        }
    }
    // ---- split-K reduction by the bulk-copy engine: rows [q R, (q + 1) R) of every CTA's partial
    // tile (R = BM / ks) are added (cp.reduce.async.bulk .add.u64) into CTA q's copy; CTA q then
    // runs the epilogue on its fully reduced slice from local shared memory ----
    const int ks = g.ks;
    cg::cluster_group cluster = cg::this_cluster();
    const int rank = (int)cluster.block_rank();
    if (PSML_TCSEG_RED == 1 && ks > 1) {
        cluster.sync();   // every CTA's partial tile written
        TS(6);
        const uint32_t rb = smem_u32(red);
        if (tid < NT) switch (ks) {
        case 2: slice_sum_store<2>(a, p, m0, n0, rank, rb, zpre); break;
        case 4: slice_sum_store<4>(a, p, m0, n0, rank, rb, zpre); break;
        case 8: slice_sum_store<8>(a, p, m0, n0, rank, rb, zpre); break;
        default: slice_sum_store<16>(a, p, m0, n0, rank, rb, zpre); break;
        }
    } else {
        const uint32_t slice_bytes = (uint32_t)(BM / ks) * RED_PITCH * 8;
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // red writes -> bulk-copy proxy
        if (tid == 0 && ks > 1)
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(rbar)),
                         "r"((uint32_t)(ks - 1) * slice_bytes)
                         : "memory");
        fence_before();
        cluster.sync();   // every partial written, every receiver armed, every pipeline idle
        TS(6);
        if (tid == 0 && ks > 1) {
            const uint32_t base = smem_u32(red), bar = smem_u32(rbar);
            for (int q = 0; q < ks; ++q) {
                if (q == rank) continue;
                const uint32_t src = base + (uint32_t)q * slice_bytes;
                uint32_t dst, dbar;
                asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(dst) : "r"(src), "r"(q));
                asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(dbar) : "r"(bar), "r"(q));
                asm volatile(
                    "cp.reduce.async.bulk.shared::cluster.shared::cta.mbarrier::complete_tx::bytes.add.u64 [%0], [%1], "
                    "%2, [%3];" ::"r"(dst),
                    "r"(src), "r"(slice_bytes), "r"(dbar)
                    : "memory");
            }
        }
        if (ks > 1) mbar_wait(smem_u32(rbar), 0);
        if (tid < NT) switch (ks) {
        case 1: slice_store<1>(a, p, m0, n0, rank, red, zpre); break;
        case 2: slice_store<2>(a, p, m0, n0, rank, red, zpre); break;
        case 4: slice_store<4>(a, p, m0, n0, rank, red, zpre); break;
        case 8: slice_store<8>(a, p, m0, n0, rank, red, zpre); break;
        default: slice_store<16>(a, p, m0, n0, rank, red, zpre); break;
        }
    }
    cluster.sync();   // peers' shared memory stays alive until every CTA has read it
    TS(7);
    if (warp == 1) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem));
    TS(8);
#ifdef TCSEG_TIMING
    if (tid == 0 && (blockIdx.x == 0 || blockIdx.x == gridDim.x - 1) && blockIdx.z < 2)
        printf("tcseg grid %d blk %d z %d nblk %d: prologue %llu load0 %llu mma %llu accum %llu red %llu reduce %llu end %llu total %llu ns\n",
               (int)gridDim.x, (int)blockIdx.x, (int)blockIdx.z, nblk, ts[1] - ts[0], ts[2] - ts[1], ts[3] - ts[2],
               ts[4] - ts[3], ts[6] - ts[4], ts[7] - ts[6], ts[8] - ts[7], ts[8] - ts[0]);
#endif
}

}  // namespace tcseg

bool tc_seg_forced() { return cur_opts().seg_backend == 2; }   // psml_options.seg_backend

bool tc_seg_enabled() {
    static int sm100 = -1;   // a device property, not an option
    if (sm100 < 0) {
        int dev = 0, maj = 0, mnr = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&maj, cudaDevAttrComputeCapabilityMajor, dev);
        cudaDeviceGetAttribute(&mnr, cudaDevAttrComputeCapabilityMinor, dev);
        cudaGetLastError();
        sm100 = (maj == 10 && mnr == 0) ? 1 : 0;
    }
    return sm100 == 1 && cur_opts().seg_backend != 1;   // tcgen05 needs sm_100
}

// psml_options.pdl = 0 disables programmatic dependent launch of the GEMMs after their producers.
bool pdl_enabled() { return cur_opts().pdl != 0; }

psml_status tc_seg_group(const SegArgs<uint64_t> *jobs, int njobs, cudaStream_t stream, int sm_count) {
    using namespace tcseg;
    if (njobs < 1 || njobs > SEG_MAX_JOBS) return fail(PSML_ERR_INVALID, "tc seg group: 1..4 jobs");
    static int attr_done = 0;
    static int max_ks = 8;
    if (!attr_done) {
        PSML_CUDA_TRY(cudaFuncSetAttribute(tc_seg_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)SMEM_BYTES));
        if (cudaFuncSetAttribute(tc_seg_kernel, cudaFuncAttributeNonPortableClusterSizeAllowed, 1) == cudaSuccess) {
            cudaLaunchConfig_t q = {};
            q.gridDim = dim3(MAX_KS, 1, MAX_KS);
            q.blockDim = dim3(NTH);
            q.dynamicSmemBytes = SMEM_BYTES;
            cudaLaunchAttribute at[1];
            at[0].id = cudaLaunchAttributeClusterDimension;
            at[0].val.clusterDim.x = 1; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = MAX_KS;
            q.attrs = at;
            q.numAttrs = 1;
            int n = 0;
            if (cudaOccupancyMaxActiveClusters(&n, tc_seg_kernel, &q) == cudaSuccess && n >= 4) max_ks = MAX_KS;
        }
        cudaGetLastError();
        attr_done = 1;
    }
    Group g{};
    int64_t tiles = 0;
    int nkb_max = 1;
    double work = 0;
    for (int q = 0; q < njobs; ++q) {
        const SegArgs<uint64_t> &j = jobs[q];
        if (2 * j.K > 16384) return fail(PSML_ERR_UNSUPPORTED, "tc seg: K' > 16384 per product");
        g.j[q] = j;
        g.tiles_m[q] = (int)((j.M + BM - 1) / BM);
        g.tiles_n[q] = (int)((j.N + BN - 1) / BN);
        g.tile_begin[q] = tiles;
        tiles += (int64_t)g.tiles_m[q] * g.tiles_n[q] * j.nparty;
        nkb_max = std::max(nkb_max, (int)((2 * j.K + BK - 1) / BK));
        work += (double)j.M * j.N * 2 * j.K * j.nparty;
    }
    g.tile_begin[njobs] = tiles;
    g.njobs = njobs;
    // K split: double ks while the grid stays within 1/PSML_TCSEG_FILL of the SMs (default 2: the
    // rest stays with the dealer branch) and each split keeps >= 2 K blocks
    const int fill = PSML_TCSEG_FILL;
    int ks = 1;
    while (ks < max_ks && tiles * ks * 2 * fill <= 2 * sm_count && nkb_max >= ks * 2) ks *= 2;
    g.ks = ks;
    for (int q = 0; q < njobs; ++q) {
        const int nkb = (int)((2 * jobs[q].K + BK - 1) / BK);
        g.kb_per_split[q] = (nkb + ks - 1) / ks;
    }
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)tiles, 1, (unsigned)ks);
    cfg.blockDim = dim3(NTH);
    cfg.dynamicSmemBytes = SMEM_BYTES;
    cfg.stream = stream;
    cudaLaunchAttribute attr[3];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = 1; attr[0].val.clusterDim.y = 1; attr[0].val.clusterDim.z = (unsigned)ks;
    attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[1].val.programmaticStreamSerializationAllowed = pdl_enabled() ? 1 : 0;
    cfg.attrs = attr;
    cfg.numAttrs = 2;
    if (cudaEvent_t ev = take_launch_event()) {   // fires once every CTA of this grid is resident
        attr[2].id = cudaLaunchAttributeLaunchCompletionEvent;
        attr[2].val.launchCompletionEvent.event = ev;
        attr[2].val.launchCompletionEvent.flags = 0;
        cfg.numAttrs = 3;
    }
    ProfScope prof(PROF_TC, stream, work);
    PSML_CUDA_TRY(cudaLaunchKernelEx(&cfg, tcseg::tc_seg_kernel, g));
    g_launches.fetch_add(1, std::memory_order_relaxed);
    return PSML_OK;
}

}  // namespace psml
