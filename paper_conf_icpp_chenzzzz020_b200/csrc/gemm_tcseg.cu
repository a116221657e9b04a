// gemm_tcseg.cu -- the opened Beaver product of the training step (Eq. 8:
// C_p = [X_p | E] . [F ; V_p] + Z_p, then SecureML truncation) on the tcgen05 tensor cores, for
// the small products of the paper's workloads (MLP 128 x 784 x 128 ... 784 x 128 x 128).
//
// Same exact limb decomposition as gemm_tc.cu (8-bit limbs, the 36 limb pairs p + q < 8 of Z_2^64
// as tcgen05.mma.kind::i8 into 8 per-shift s32 TMEM accumulators S_s, result sum_s S_s 2^{8s}),
// but built for products whose whole operand set is a few MB: there is NO separate limb-split
// pass through HBM.  The CTA's 8 producer warps load the uint64 operand words of K block i + 2
// straight from the producers' outputs (L2-resident) into registers (32-byte loads: a warp reads
// four whole 256-byte rows of A per instruction) while they split block i into limb bytes (a 4 x 4
// byte transpose per 4 words: 2 PRMT per limb word) and store them into shared memory in the UMMA
// K-major no-swizzle canonical layout; warp 8 issues the block's limb-pair MMAs (the B planes of
// one A limb as one N <= 256 operand: 12 MMAs per block) as soon as the stage's `full` barrier
// completes (3-stage ring; the commit of a stage's MMAs frees it).  Per 128 x 64 x 32 block a CTA
// moves 48 KB of limb planes into shared memory and the MMAs read 120 KB back (A 12 x 4 KB, B
// 36 x 2 KB): 168 KB at 128 B/clk is 1.3 us -- the kernel's shared-memory roofline (measured
// 1.4 us per block with every SM busy).
// K is split over the ks CTAs of a (1, 1, ks) thread-block cluster: each CTA turns its
// accumulators into uint64 partials (exact mod 2^64, K' per CTA <= 2^14 keeps S_0..S_3 exact),
// the partial tiles are summed through distributed shared memory, and each CTA runs the epilogue
// (+ Z_p, truncation, store) on 1/ks of the tile.  Ring addition is exact, so the result is
// bit-identical to the CUDA-core seg_gemm_kernel (tested).
// segs = 1 runs the plain product X . F (K' = K, no Z): psml_ring_gemm at small n (config 5).
#include <cooperative_groups.h>

#include "engine.h"
#include "fused.cuh"

namespace psml {
namespace tcseg {

constexpr int BM = 128, BN = 64, BK = 32, NT = 256, LMAX = 8;
#ifndef TCSEG_STAGES
#define TCSEG_STAGES 3   // limb-stage ring (same box: 4 -> 3 stages 1024^3 55.3 -> 53.2 us, step unchanged; 2 slower e2e)
#endif
constexpr int STAGES = TCSEG_STAGES;
constexpr int NTH = NT + 32;   // NT producer threads (loads, limb split, epilogue) + the MMA warp
constexpr int A_TILE = BM * BK;                        // bytes per limb plane of one A block
constexpr int B_TILE = BN * BK;                        // bytes per limb plane of one B block
constexpr int STAGE_BYTES = LMAX * (A_TILE + B_TILE);  // stage stride: 48 KB (l = 64: 8 limb planes each)
constexpr int RED_PITCH = BN + 1;                      // words per row of the reduction tile
constexpr int PIPE_BYTES = STAGES * STAGE_BYTES;
static_assert(BM * RED_PITCH * 8 <= PIPE_BYTES, "reduction tile must fit the pipeline region");
constexpr size_t SMEM_BYTES = PIPE_BYTES + 8 * (2 * STAGES + 2) + 16;   // > 114 KB: one CTA per SM
constexpr int MAX_KS = 16;

template <typename T>
struct Group {
    SegArgs<T> j[SEG_MAX_JOBS];
    int64_t tile_begin[SEG_MAX_JOBS + 1];
    int tiles_n[SEG_MAX_JOBS], tiles_m[SEG_MAX_JOBS];
    int kb_per_split[SEG_MAX_JOBS];
    int njobs, ks;
    int segs;   // 2: the Beaver product [X_p | E] . [F ; V_p] (K' = 2K); 1: the plain product X . F (K' = K)
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
// limb words of 4 consecutive ring elements: out[p] = bytes p of v0..v3 (p < sizeof(T))
__device__ __forceinline__ void limbs4(const uint64_t *v, uint32_t out[8]) {
    bt4((uint32_t)v[0], (uint32_t)v[1], (uint32_t)v[2], (uint32_t)v[3], out);
    bt4((uint32_t)(v[0] >> 32), (uint32_t)(v[1] >> 32), (uint32_t)(v[2] >> 32), (uint32_t)(v[3] >> 32), out + 4);
}
__device__ __forceinline__ void limbs4(const uint32_t *v, uint32_t out[4]) { bt4(v[0], v[1], v[2], v[3], out); }

__device__ __forceinline__ uint64_t ldg(const uint64_t *p) { return __ldg((const unsigned long long *)p); }
__device__ __forceinline__ uint32_t ldg(const uint32_t *p) { return __ldg((const unsigned int *)p); }
// 4 consecutive words (32 B for l = 64, 16 B for l = 32; aligned)
__device__ __forceinline__ void ld4(const uint64_t *p, uint64_t *v) {
    asm volatile("ld.global.nc.v4.u64 {%0, %1, %2, %3}, [%4];" : "=l"(v[0]), "=l"(v[1]), "=l"(v[2]), "=l"(v[3]) : "l"(p));
}
__device__ __forceinline__ void ld4(const uint32_t *p, uint32_t *v) {
    const uint4 q = __ldg((const uint4 *)p);
    v[0] = q.x; v[1] = q.y; v[2] = q.z; v[3] = q.w;
}
// one A unit of UW consecutive words in one load: 32 B (4 x u64 or 8 x u32; aligned)
__device__ __forceinline__ void ld_unit(const uint64_t *p, uint64_t *v) { ld4(p, v); }
__device__ __forceinline__ void ld_unit(const uint32_t *p, uint32_t *v) {
    uint64_t a, b, c, d;
    asm volatile("ld.global.nc.v4.u64 {%0, %1, %2, %3}, [%4];" : "=l"(a), "=l"(b), "=l"(c), "=l"(d) : "l"(p));
    v[0] = (uint32_t)a; v[1] = (uint32_t)(a >> 32); v[2] = (uint32_t)b; v[3] = (uint32_t)(b >> 32);
    v[4] = (uint32_t)c; v[5] = (uint32_t)(c >> 32); v[6] = (uint32_t)d; v[7] = (uint32_t)(d >> 32);
}
__device__ __forceinline__ uint64_t ld_dsmem(uint32_t a, uint64_t *) {
    uint64_t v;
    asm volatile("ld.shared::cluster.u64 %0, [%1];" : "=l"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ uint32_t ld_dsmem(uint32_t a, uint32_t *) {
    uint32_t v;
    asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(v) : "r"(a));
    return v;
}
constexpr int ZPF = 8;   // epilogue Z words prefetched per thread (ks >= 4)
#ifndef TCSEG_EPI_UNROLL
#define TCSEG_EPI_UNROLL 4    // epilogue loop unrolling for ks <= 2 (code size vs instruction-level parallelism)
#endif

// Epilogue of this CTA's reduced slice (rows [rank R, (rank + 1) R) of the tile, R = BM / KS):
// thread tid owns elements e = rank * PER + tid + NT * i (i < NEL); + Z_p, truncation, store.
template <typename T, int KS>
__device__ __forceinline__ void slice_store(const SegArgs<T> &a, int p, int64_t m0, int64_t n0, int rank,
                                            const T *red, const T zpre[ZPF]) {
    constexpr int PER = BM * BN / KS, NEL = PER / NT, UNR = NEL <= ZPF ? NEL : TCSEG_EPI_UNROLL;
    const int tid = threadIdx.x, party = a.party[p];
#pragma unroll (UNR)
    for (int i = 0; i < NEL; ++i) {
        const int e = rank * PER + tid + NT * i;
        const int r = e / BN, c = e % BN;
        const int64_t m = m0 + r, n = n0 + c;
        const int64_t off = (m < a.M ? m : a.M - 1) * a.N + (n < a.N ? n : a.N - 1);
        const T z = !a.Z[p] ? 0 : NEL <= ZPF ? zpre[i < ZPF ? i : 0] : ldg(a.Z[p] + off);
        const T sum = red[r * RED_PITCH + c];
        if (m < a.M && n < a.N) a.C[p][off] = trunc_share<T>(sum + z, party, a.trunc);
    }
}

// The same epilogue, summing the slice's rows straight out of every cluster CTA's partial tile
// (ld.shared::cluster: distributed shared memory reads, KS loads per element in flight).
template <typename T, int KS>
__device__ __forceinline__ void slice_sum_store(const SegArgs<T> &a, int p, int64_t m0, int64_t n0, int rank,
                                                uint32_t red_u32, const T zpre[ZPF]) {
    constexpr int PER = BM * BN / KS, NEL = PER / NT, UNR = NEL <= ZPF ? NEL : TCSEG_EPI_UNROLL;
    const int tid = threadIdx.x, party = a.party[p];
    uint32_t peer[KS];
#pragma unroll
    for (int q = 0; q < KS; ++q) asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(peer[q]) : "r"(red_u32), "r"(q));
#pragma unroll (UNR)
    for (int i = 0; i < NEL; ++i) {
        const int e = rank * PER + tid + NT * i;
        const int r = e / BN, c = e % BN;
        const uint32_t off = (uint32_t)(r * RED_PITCH + c) * (uint32_t)sizeof(T);
        T part[KS];
#pragma unroll
        for (int q = 0; q < KS; ++q) part[q] = ld_dsmem(peer[q] + off, (T *)nullptr);
        T sum = 0;
#pragma unroll
        for (int q = 0; q < KS; ++q) sum += part[q];
        const int64_t m = m0 + r, n = n0 + c;
        const int64_t o = (m < a.M ? m : a.M - 1) * a.N + (n < a.N ? n : a.N - 1);
        const T z = !a.Z[p] ? 0 : NEL <= ZPF ? zpre[i < ZPF ? i : 0] : ldg(a.Z[p] + o);
        if (m < a.M && n < a.N) a.C[p][o] = trunc_share<T>(sum + z, party, a.trunc);
    }
}


// grid (total tiles, 1, ks), cluster (1, 1, ks), NTH threads, SMEM_BYTES dynamic shared memory.
// Warps 0-7 load the operand words into registers and split them into limb planes; warp 8 issues
// the MMAs of each limb stage as soon as its `full` barrier completes, so the tensor core works
// on block i while the producers split block i + 1.
template <typename T>
__global__ void __launch_bounds__(NTH, 1) tc_seg_kernel(const __grid_constant__ Group<T> g) {
    constexpr int L = (int)sizeof(T);   // 8-bit limbs per ring element
#ifndef TCSEG_PD64
#define TCSEG_PD64 2
#endif
#ifndef TCSEG_PD32
#define TCSEG_PD32 2
#endif
    constexpr int PD = L == 8 ? TCSEG_PD64 : TCSEG_PD32;   // K blocks of operand words in flight per producer
    namespace cg = cooperative_groups;
    extern __shared__ __align__(1024) uint8_t smem[];
    uint64_t *empty = (uint64_t *)(smem + PIPE_BYTES);   // limb stage free (MMAs of its block done)
    uint64_t *full = empty + STAGES;                      // limb stage written by all NT producers
    uint64_t *accum = full + STAGES;
    uint32_t *tmem_slot = (uint32_t *)(accum + 1);
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
    const SegArgs<T> &a = g.j[jb];
    const int64_t tt = t - g.tile_begin[jb];
    const int64_t per_party = (int64_t)g.tiles_m[jb] * g.tiles_n[jb];
    const int p = (int)(tt / per_party);
    const int64_t tp = tt - p * per_party;
    const int64_t m0 = (tp / g.tiles_n[jb]) * BM, n0 = (tp % g.tiles_n[jb]) * BN;
    const int64_t M = a.M, N = a.N, K = a.K, Kext = g.segs * K;
    const int nkb = (int)((Kext + BK - 1) / BK);
    const int kb0 = (int)blockIdx.z * g.kb_per_split[jb];
    const int kb1 = min(kb0 + g.kb_per_split[jb], nkb);
    const int nblk = kb1 > kb0 ? kb1 - kb0 : 0;
    const T *Xp = a.X[p], *Ep = a.E, *Fp = a.F, *Vp = a.V[p];

    if (tid == 0) {
        for (int s = 0; s < STAGES; ++s) {
            mbar_init(smem_u32(&empty[s]), 1);
            mbar_init(smem_u32(&full[s]), NT);
        }
        mbar_init(smem_u32(accum), 1);
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
    T zpre[ZPF];
    {
        const int ks = g.ks, nel = (BM * BN) / ks / NT;
#pragma unroll
        for (int i = 0; i < ZPF; ++i) {
            zpre[i] = 0;
            if (nel <= ZPF && i < nel && tid < NT && a.Z[p]) {
                const int e = (int)blockIdx.z * (nel * NT) + tid + NT * i;
                const int64_t m = m0 + e / BN, n = n0 + e % BN;
                zpre[i] = ldg(a.Z[p] + (m < M ? m : M - 1) * N + (n < N ? n : N - 1));
            }
        }
    }

    // B unit of a producer thread: column bn, 8-k quarter bq of each K block
    const int bn = tid & 63, bq = tid >> 6;
    const int b_off = (((bn >> 3) * 2 + (bq >> 1)) * 128) + (bn & 7) * 16 + (bq & 1) * 8;

    // Programmatic dependent launch: everything above (barriers, TMEM, Z prefetch -- the dealer's
    // output, complete before the predecessor kernel started) overlapped the predecessor; the
    // operands X_p / E / F it produces are read only after this wait.
    pdl_trigger();
    pdl_wait();
    if (warp < NT / 32) {   // producers
        // Each thread owns four A units (row u >> 3, 4-k chunk u & 7 of units u = tid + NT i: a warp
        // reads 4 whole 256-byte rows per instruction, one 32-byte load per unit) and one B unit
        // (column bn, 8-k quarter bq) of every K block, and loads their words straight into
        // registers two blocks ahead (double-buffered register sets): a block's words pass through
        // shared memory once -- as limb planes -- instead of raw words in + out + limb planes.
        const int64_t bnn = n0 + bn;
        const bool bcol = bnn < N;
        // an A unit is UW consecutive k of one row = 32 bytes (4 words at l = 64, 8 at l = 32):
        // NU units per thread, UPR units per 32-k row of the block
        constexpr int UW = 32 / (int)sizeof(T), NU = 16 / UW, UPR = BK / UW;
        auto alv = [](const void *q) { return ((uintptr_t)q & 31) == 0; };
        const bool a32 = (K % UW) == 0 && alv(Xp) && alv(Ep);
        // interior blocks (every row / column inside, the 32 k inside one segment) take a fast path:
        // precomputed row offsets, no bounds checks, one address add per load
        const bool rows_full = m0 + BM <= M && a32, cols_full = n0 + BN <= N;
        int64_t rowoff[NU];
#pragma unroll
        for (int i = 0; i < NU; ++i) {
            const int u = tid + NT * i;
            rowoff[i] = (m0 + u / UPR) * K + UW * (u % UPR);
        }
        const int64_t colbase = (int64_t)(8 * bq) * N + bnn;
        auto load = [&](int kb, T (&va)[16], T (&vb)[8]) {
            const int64_t k0 = (int64_t)kb * BK;
            const bool one_seg = k0 + BK <= K || (k0 >= K && k0 + BK <= Kext);
            if (rows_full && one_seg) {
                const T *sb = k0 < K ? Xp + k0 : Ep + (k0 - K);
#pragma unroll
                for (int i = 0; i < NU; ++i) ld_unit(sb + rowoff[i], va + UW * i);
            } else {
#pragma unroll
                for (int i = 0; i < NU; ++i) {
                    const int u = tid + NT * i, row = u / UPR;
                    const int64_t m = m0 + row, k = k0 + UW * (u % UPR);
                    const int64_t mc = m < M ? m : 0;
                    if (a32) {
                        if (m < M && k < Kext) {
                            ld_unit(k < K ? Xp + mc * K + k : Ep + mc * K + (k - K), va + UW * i);
                        } else {
#pragma unroll
                            for (int j = 0; j < UW; ++j) va[UW * i + j] = 0;
                        }
                    } else {
#pragma unroll
                        for (int j = 0; j < UW; ++j) {
                            const int64_t kk = k + j;
                            va[UW * i + j] = (m < M && kk < Kext) ? ldg(kk < K ? Xp + mc * K + kk : Ep + mc * K + (kk - K)) : 0;
                        }
                    }
                }
            }
            if (cols_full && one_seg) {
                const T *bb = (k0 < K ? Fp + k0 * N : Vp + (k0 - K) * N) + colbase;
#pragma unroll
                for (int j = 0; j < 8; ++j) vb[j] = ldg(bb + j * N);
            } else {
                const int64_t kbq = k0 + 8 * bq;
#pragma unroll
                for (int j = 0; j < 8; ++j) {
                    const int64_t k = kbq + j;
                    vb[j] = (bcol && k < Kext) ? ldg(k < K ? Fp + k * N + bnn : Vp + (k - K) * N + bnn) : 0;
                }
            }
        };
        auto stash_regs = [&](int st, const T (&va)[16], const T (&vb)[8]) {
            uint8_t *sa = smem + st * STAGE_BYTES, *sb = sa + L * A_TILE;
#pragma unroll
            for (int i = 0; i < NU; ++i) {
                const int u = tid + NT * i, row = u / UPR, k = UW * (u % UPR);
                // the unit's k range inside the 16-byte core-matrix row of each limb plane
                const int off = (((row >> 3) * 2 + (k >> 4)) * 128) + (row & 7) * 16 + (k & 15);
                if constexpr (UW == 4) {
                    uint32_t w[L];
                    limbs4(va + UW * i, w);
#pragma unroll
                    for (int l = 0; l < L; ++l) *(uint32_t *)(sa + l * A_TILE + off) = w[l];
                } else {   // 8 k: two limb words per plane, one 8-byte store
                    uint32_t w0[L], w1[L];
                    limbs4(va + UW * i, w0);
                    limbs4(va + UW * i + 4, w1);
#pragma unroll
                    for (int l = 0; l < L; ++l) *(uint2 *)(sa + l * A_TILE + off) = make_uint2(w0[l], w1[l]);
                }
            }
            uint32_t u[2][L];
            limbs4(vb, u[0]);
            limbs4(vb + 4, u[1]);
#pragma unroll
            for (int l = 0; l < L; ++l) *(uint2 *)(sb + l * B_TILE + b_off) = make_uint2(u[0][l], u[1][l]);
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // generic writes -> tensor core
        };
        // PD register sets: block i + PD is loaded as soon as block i is stashed
        T ra[PD][16], rb[PD][8];
#pragma unroll
        for (int d = 0; d < PD; ++d)
            if (d < nblk) load(kb0 + d, ra[d], rb[d]);
        TS(2);
        auto step = [&](int i, T (&va)[16], T (&vb)[8]) {
            const int st = i % STAGES;
            if (i >= STAGES) mbar_wait(smem_u32(&empty[st]), (uint32_t)((i / STAGES - 1) & 1));
            stash_regs(st, va, vb);
            asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&full[st])) : "memory");
            if (i + PD < nblk) load(kb0 + i + PD, va, vb);
        };
        for (int i = 0; i < nblk; i += PD) {
#pragma unroll
            for (int d = 0; d < PD; ++d)
                if (i + d < nblk) step(i + d, ra[d], rb[d]);
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

    // ---- partial tile: sum_s S_s 2^{8s} (mod 2^l, exact) -> reduction buffer ----
    T *red = (T *)smem;   // the pipeline region is idle once `accum` completes
    mbar_wait(smem_u32(accum), 0);
    TS(4);
    fence_after();
    if (warp < NT / 32) {   // warps w and w + 4 share TMEM lanes 32 (w % 4) ..; each drains half the columns
        const int row = (warp & 3) * 32 + lane;
        const uint32_t lane_base = tmem + ((uint32_t)((warp & 3) * 32) << 16);
#pragma unroll 1
        for (int j0 = (warp >> 2) * (BN / 2); j0 < (warp >> 2) * (BN / 2) + BN / 2; j0 += 16) {
            T acc[16];
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
                        for (int j = 0; j < 16; ++j) acc[j] += (T)r[16 * u + j] << (8 * (s0 + u));
                }
            }
#pragma unroll
            for (int j = 0; j < 16; ++j) red[row * RED_PITCH + j0 + j] = acc[j];
        }
    }
    // ---- split-K reduction: each CTA sums rows [rank R, (rank + 1) R) (R = BM / ks) of every
    // cluster CTA's partial tile straight out of their shared memory (DSMEM reads) and runs the
    // epilogue on that slice ----
    const int ks = g.ks;
    cg::cluster_group cluster = cg::this_cluster();
    const int rank = (int)cluster.block_rank();
    cluster.sync();   // every CTA's partial tile written
    TS(6);
    if (tid < NT) switch (ks) {
    case 1: slice_store<T, 1>(a, p, m0, n0, rank, red, zpre); break;
    case 2: slice_sum_store<T, 2>(a, p, m0, n0, rank, smem_u32(red), zpre); break;
    case 4: slice_sum_store<T, 4>(a, p, m0, n0, rank, smem_u32(red), zpre); break;
    case 8: slice_sum_store<T, 8>(a, p, m0, n0, rank, smem_u32(red), zpre); break;
    default: slice_sum_store<T, 16>(a, p, m0, n0, rank, smem_u32(red), zpre); break;
    }
    cluster.sync();   // peers' shared memory stays alive until every CTA has read it
    TS(7);
    if (warp == 1) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem));
    TS(8);
#ifdef TCSEG_TIMING_ALL
    if (tid == 0) {
        uint32_t smid;
        asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
        printf("tcsegall %d %d %u %llu %llu\n", (int)blockIdx.x, (int)blockIdx.z, smid, ts[0], ts[8]);
    }
#elif defined(TCSEG_TIMING)
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

template <typename T>
static psml_status tc_seg_group_t(const SegArgs<T> *jobs, int njobs, cudaStream_t stream, int sm_count, int segs,
                                  int fill) {
    using namespace tcseg;
    if (njobs < 1 || njobs > SEG_MAX_JOBS) return fail(PSML_ERR_INVALID, "tc seg group: 1..4 jobs");
    static int attr_done = 0;
    static int max_ks = 8;
    if (!attr_done) {
        PSML_CUDA_TRY(cudaFuncSetAttribute(tcseg::tc_seg_kernel<T>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)SMEM_BYTES));
        if (cudaFuncSetAttribute(tcseg::tc_seg_kernel<T>, cudaFuncAttributeNonPortableClusterSizeAllowed, 1) == cudaSuccess) {
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
            if (cudaOccupancyMaxActiveClusters(&n, tcseg::tc_seg_kernel<T>, &q) == cudaSuccess && n >= 4) max_ks = MAX_KS;
        }
        cudaGetLastError();
        attr_done = 1;
    }
    Group<T> g{};
    int64_t tiles = 0;
    int nkb_max = 1;
    double work = 0;
    for (int q = 0; q < njobs; ++q) {
        const SegArgs<T> &j = jobs[q];
        // l = 64: K' <= 2^14 per CTA keeps S_0..S_3 exact in s32 (every shift wraps harmlessly mod 2^32 at l = 32)
        if (sizeof(T) == 8 && segs * j.K > 16384) return fail(PSML_ERR_UNSUPPORTED, "tc seg: K' > 16384 per product");
        g.j[q] = j;
        g.tiles_m[q] = (int)((j.M + BM - 1) / BM);
        g.tiles_n[q] = (int)((j.N + BN - 1) / BN);
        g.tile_begin[q] = tiles;
        tiles += (int64_t)g.tiles_m[q] * g.tiles_n[q] * j.nparty;
        nkb_max = std::max(nkb_max, (int)((segs * j.K + BK - 1) / BK));
        work += (double)j.M * j.N * segs * j.K * j.nparty;
    }
    g.tile_begin[njobs] = tiles;
    g.njobs = njobs;
    g.segs = segs;
    // K split: double ks while the grid stays within 2/fill of the SMs (training step, fill = 2: the
    // rest stays with the dealer branch; fill = 0: stand-alone products, one wave) and each split
    // keeps >= 2 K blocks
    int ks = 1;
    if (fill > 0) {   // training step (measured: up to 2 sm_count / fill CTAs)
        while (ks < max_ks && tiles * ks * 2 * fill <= 2 * sm_count && nkb_max >= ks * 2) ks *= 2;
    } else {          // stand-alone: the whole grid in one wave of one-CTA-per-SM clusters
        while (ks < max_ks && tiles * ks * 2 <= sm_count && nkb_max >= ks * 2) ks *= 2;
    }
    g.ks = ks;
    for (int q = 0; q < njobs; ++q) {
        const int nkb = (int)((segs * jobs[q].K + BK - 1) / BK);
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
    PSML_CUDA_TRY(cudaLaunchKernelEx(&cfg, tcseg::tc_seg_kernel<T>, g));
    g_launches.fetch_add(1, std::memory_order_relaxed);
    return PSML_OK;
}

psml_status tc_seg_group(const SegArgs<uint64_t> *jobs, int njobs, cudaStream_t stream, int sm_count, int segs,
                         int fill) {
    return tc_seg_group_t<uint64_t>(jobs, njobs, stream, sm_count, segs, fill);
}

// ------------------------------------------------------------------------------------------------
// Stand-alone products on the same kernel (BASELINE config 5 at n <= 2048, psml_ring_gemm and the
// co-resident psml_secure_matmul): the limb-plane kernels of gemm_tc.cu need a split pass, a
// split-K memset and a finalize launch around a grid of few 128 x 128 tiles at these sizes; here
// one launch (plain) or two (Beaver: one mask + open pass, then the Eq. 8 product) cover them,
// with the K split over a cluster filling the whole GPU.
// ------------------------------------------------------------------------------------------------
bool tc_seg_small(int l, int64_t M, int64_t Kext, int64_t N, int nparty, int sm_count) {
    const int mode = cur_opts().tc_small;   // psml_options.tc_small
    if (mode == 0 || !tc_seg_enabled() || (l == 64 && Kext > 16384) || M <= 0 || N <= 0) return false;
    if (mode == 2) return true;
    // auto: the output tiles fit one wave, two for l = 64 (measured, tools/tc_small_ab.py and the
    // config-5 sweep: 512^3 plain 44 -> 18.5 us, 1024^3 plain 93 -> 52 us; Beaver 1024^3 (256 tiles)
    // l = 64 224 -> 204 us, but l = 32 112 us on the limb planes vs 142; 2048^3 plain l = 64 280 us on
    // the limb planes vs 330)
    using namespace tcseg;
    const int64_t tiles = ((M + BM - 1) / BM) * ((N + BN - 1) / BN) * nparty;
    return tiles <= (l == 64 ? 2 : 1) * (int64_t)sm_count;
}

template <typename T>
psml_status tc_seg_plain(const T *A, const T *B, int64_t M, int64_t K, int64_t N, T *C, cudaStream_t s, int sm_count) {
    SegArgs<T> a{};
    a.X[0] = A; a.F = B; a.C[0] = C;
    a.M = M; a.N = N; a.K = K; a.trunc = 0; a.nparty = 1;
    return tc_seg_group_t<T>(&a, 1, s, sm_count, 1, 0);
}

template <typename T>
size_t tc_seg_beaver_ws_bytes(int64_t M, int64_t K, int64_t N) { return sizeof(T) * (size_t)(2 * M * K + K * N) + 512; }

template <typename T>
psml_status tc_seg_beaver(const T *const A[2], const T *const B[2], const T *const U[2], const T *const V[2],
                          const T *const Z[2], int64_t M, int64_t K, int64_t N, int flags, int trunc, T *const C[2],
                          void *ws, size_t ws_bytes, cudaStream_t s, int sm_count) {
    if (ws_bytes < tc_seg_beaver_ws_bytes<T>(M, K, N)) return fail(PSML_ERR_NOMEM, "tc seg Beaver workspace too small");
    T *E = (T *)(((uintptr_t)ws + 255) & ~(uintptr_t)255), *X1 = E + M * K, *F = X1 + M * K;
    // Eqs. 4-5 for both parties in one pass: E = (A_0 - U_0) + (A_1 - U_1), X_1 = E + U_1,
    // F = (B_0 - V_0) + (B_1 - V_1) (op layouts; transposed sources through shared memory)
    OpenList<T> L{};
    const int tA = (flags & PSML_TRANS_A) ? 1 : 0, tB = (flags & PSML_TRANS_B) ? 1 : 0;
    L.j[0] = {{A[0], A[1]}, {U[0], U[1]}, E, X1, U[1], (T)1, M, K, tA};
    L.j[1] = {{B[0], B[1]}, {V[0], V[1]}, F, nullptr, nullptr, (T)1, K, N, tB};
    L.n = 2;
    L.tile_begin[0] = 0;
    L.tile_begin[1] = ((M + 31) / 32) * ((K + 31) / 32);
    L.tile_begin[2] = L.tile_begin[1] + ((K + 31) / 32) * ((N + 31) / 32);
    {
        ProfScope prof(PROF_MASK, s, 3.0 * 8 * 2 * (M * K + K * N));
        PSML_CUDA_TRY(launch_pdl(open_list_kernel<T>, dim3((unsigned)L.tile_begin[2]), dim3(32, 8), s, L));
        PSML_LAUNCH_CHECK();
    }
    // Eq. 8 (BJ form): C_p = [X_p | E] . [F ; V_p] + Z_p, X_0 = U_0, then truncation
    SegArgs<T> a{};
    a.X[0] = U[0]; a.X[1] = X1; a.E = E; a.F = F;
    for (int p = 0; p < 2; ++p) { a.V[p] = V[p]; a.Z[p] = Z[p]; a.C[p] = C[p]; a.party[p] = p; }
    a.M = M; a.N = N; a.K = K; a.trunc = trunc; a.nparty = 2;
    return tc_seg_group_t<T>(&a, 1, s, sm_count, 2, 0);
}

#define PSML_TCSEG_INST(T)                                                                                        \
    template psml_status tc_seg_plain<T>(const T *, const T *, int64_t, int64_t, int64_t, T *, cudaStream_t, int); \
    template size_t tc_seg_beaver_ws_bytes<T>(int64_t, int64_t, int64_t);                                        \
    template psml_status tc_seg_beaver<T>(const T *const[2], const T *const[2], const T *const[2], const T *const[2], \
                                          const T *const[2], int64_t, int64_t, int64_t, int, int, T *const[2], void *, \
                                          size_t, cudaStream_t, int);
PSML_TCSEG_INST(uint64_t)
PSML_TCSEG_INST(uint32_t)

}  // namespace psml
