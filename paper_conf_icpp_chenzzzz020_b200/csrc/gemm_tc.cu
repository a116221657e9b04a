// gemm_tc.cu -- exact ring GEMM in Z_{2^64} / Z_{2^32} on the 5th-generation tensor cores.
//
// Each operand word is split into 8-bit limbs (8 for l = 64, 4 for l = 32):
//     a = sum_p a_p 2^{8p},  b = sum_q b_q 2^{8q},  a.b mod 2^l = sum_{p+q < l/8} a_p b_q 2^{8(p+q)}
// so only the limb pairs with p + q < l/8 survive (36 of 64 for l = 64, 10 of 16 for l = 32).
// Every surviving pair is one tcgen05.mma.kind::i8 (u8 x u8 -> s32, no saturation) into the TMEM
// accumulator of its shift s = p + q:  S_s = sum_{p+q=s} A_p . B_q^T.  The epilogue forms
// sum_s S_s 2^{8s} mod 2^l in registers, adds the Beaver Z_i, truncates and stores.
// Exactness: S_s only matters mod 2^{l-8s}; for s >= l/8 - 4 that is <= 32 bits (int32 wrap is
// harmless), for l = 64 and s <= 3 we need (s+1) K' 255^2 < 2^32, i.e. K' <= 16512 per pass --
// larger K is split into exact chunks whose uint64 partials are added with atomics.
//
// Layout: limb planes are written by split_kernel already tiled in the
// UMMA K-major no-swizzle canonical form -- 8-row x 16-byte core matrices, K-adjacent core
// matrices 128 B apart (LBO), 8-row groups 256 B apart (SBO) -- so the (limb, row-block,
// k-block) tile of 128 (or BN) rows x 32 bytes is ONE contiguous chunk moved by a 1-D TMA bulk
// copy (cp.async.bulk, SASS UBLKCP) straight into shared memory.  No tensor maps needed.
//
// CTA (128 threads, 1 per SM): warp 0 lane 0 = TMA producer, warp 1 lane 0 = MMA issuer,
// warp 2 = TMEM allocator; all four warps run the epilogue (warp w owns TMEM lanes 32w..32w+31).
// Tile: 128 x BN (BN = 64 for l = 64: 8 shift accumulators x 64 columns = all 512 TMEM columns;
// BN = 128 for l = 32: 4 x 128).  K block 32 bytes per stage, 4 (l=64) / 6 (l=32) stages.
#ifndef PSML_TC_MINKB
#define PSML_TC_MINKB 4   // fewest K blocks per split-K slice (512^3: 50 -> 44 us vs 8)
#endif
#include "engine.h"

namespace psml {
namespace tc {

constexpr int BM = 128, BK = 32;

// ------------------------------------------------------------------------------------------------
// PTX wrappers
// ------------------------------------------------------------------------------------------------
__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
    asm volatile(
        "{\n"
        ".reg .pred P1;\n"
        "LAB_WAIT:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
        "@P1 bra DONE;\n"
        "bra LAB_WAIT;\n"
        "DONE:\n"
        "}\n" ::"r"(bar),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void *src, uint32_t bytes, uint32_t bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
                 "l"(src), "r"(bytes), "r"(bar)
                 : "memory");
}
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

__device__ __forceinline__ void tc_mma_i8(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                          uint32_t accumulate) {
    asm volatile(
        "{\n"
        ".reg .pred p;\n"
        "setp.ne.b32 p, %4, 0;\n"
        "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n"
        "}\n" ::"r"(d_tmem),
        "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
        : "memory");
}
__device__ __forceinline__ void tc_commit(uint32_t bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar) : "memory");
}
// the same bulk copy landing at the same shared-memory offset (and completing the mbarrier at the
// same offset) in every CTA of `mask` in the cluster
__device__ __forceinline__ void bulk_g2s_mc(uint32_t dst, const void *src, uint32_t bytes, uint32_t bar, uint16_t mask) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.multicast::cluster [%0], [%1], %2, [%3], %4;" ::"r"(dst),
        "l"(src), "r"(bytes), "r"(bar), "h"(mask)
        : "memory");
}
// commit arriving on the mbarrier at this offset in every CTA of `mask`
__device__ __forceinline__ void tc_commit_mc(uint32_t bar, uint16_t mask) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(bar),
                 "h"(mask)
                 : "memory");
}
__device__ __forceinline__ void cluster_sync_all() {
    asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ uint32_t cluster_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
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

// UMMA shared-memory descriptor, K-major, SWIZZLE_NONE (layout type 0), sm_100 version 1.
__device__ __forceinline__ uint64_t smem_desc(uint32_t addr, uint32_t lbo, uint32_t sbo) {
    return (uint64_t)((addr >> 4) & 0x3FFFu) | ((uint64_t)((lbo >> 4) & 0x3FFFu) << 16) |
           ((uint64_t)((sbo >> 4) & 0x3FFFu) << 32) | (1ull << 46);
}

// Instruction descriptor kind::i8: D s32 (c_format 2), A/B u8 (format 0), K-major, M=128, N.
__host__ __device__ constexpr uint32_t idesc_i8(int M, int N) {
    return (2u << 4) | (0u << 7) | (0u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}

// ------------------------------------------------------------------------------------------------
// limb split into the tiled canonical layout
// ------------------------------------------------------------------------------------------------
struct SplitJob {
    const void *s0, *s1, *s2;  // summed sources (nullable); A-type: rows x kcols; B-type: kcols x rows
    uint8_t *dst;              // tiled output; limb p at dst + p * limb_stride
    int64_t rows, kcols;       // logical extent
    int64_t rows_pad, k_pad;   // padded to the tile rows / BK
    int rt;                    // tile rows: 128 (A operand) or BN (B operand)
    int btype;                 // 0: source row-major rows x kcols; 1: source row-major kcols x rows
};
struct SplitJobs {
    SplitJob j[6];
    int count;
};

template <typename T, int L>
__global__ void __launch_bounds__(256) split_kernel(SplitJobs jobs) {
    const SplitJob J = jobs.j[blockIdx.y];
    const int64_t nkb = J.k_pad / BK;
    const int64_t units = J.rows_pad * (J.k_pad / 16);
    const int64_t limb_stride = J.rows_pad * J.k_pad;
    const int G = J.rt / 8;
    const T *s0 = (const T *)J.s0, *s1 = (const T *)J.s1, *s2 = (const T *)J.s2;
    for (int64_t u = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; u < units; u += (int64_t)gridDim.x * blockDim.x) {
        int64_t row, kb;
        int c, g, r8;
        if (!J.btype) {  // order (rb, kb, g, c, r8): a warp writes 512 contiguous bytes per limb
            r8 = (int)(u & 7);
            int64_t t = u >> 3;
            c = (int)(t & 1);
            t >>= 1;
            g = (int)(t % G);
            t /= G;
            kb = t % nkb;
            const int64_t rb = t / nkb;
            row = rb * J.rt + g * 8 + r8;
        } else {         // order (rb, kb, c, g, r8): a warp reads 32 consecutive source columns
            const int rr = (int)(u % J.rt);
            int64_t t = u / J.rt;
            c = (int)(t & 1);
            t >>= 1;
            kb = t % nkb;
            const int64_t rb = t / nkb;
            g = rr / 8;
            r8 = rr % 8;
            row = rb * J.rt + rr;
        }
        const int64_t k0 = kb * BK + c * 16;
        T v[16];
#pragma unroll
        for (int j = 0; j < 16; ++j) {
            const int64_t k = k0 + j;
            T x = 0;
            if (row < J.rows && k < J.kcols) {
                const int64_t idx = J.btype ? k * J.rows + row : row * J.kcols + k;
                if (s0) x += s0[idx];
                if (s1) x += s1[idx];
                if (s2) x += s2[idx];
            }
            v[j] = x;
        }
        const int64_t rb = row / J.rt;
        const int64_t off = (((rb * nkb + kb) * G + g) * 2 + c) * 128 + (int64_t)r8 * 16;
#pragma unroll
        for (int p = 0; p < L; ++p) {
            uint32_t w[4];
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                uint32_t b0 = (uint32_t)(v[4 * q + 0] >> (8 * p)) & 0xFF, b1 = (uint32_t)(v[4 * q + 1] >> (8 * p)) & 0xFF;
                uint32_t b2 = (uint32_t)(v[4 * q + 2] >> (8 * p)) & 0xFF, b3 = (uint32_t)(v[4 * q + 3] >> (8 * p)) & 0xFF;
                w[q] = b0 | (b1 << 8) | (b2 << 16) | (b3 << 24);
            }
            *(uint4 *)(J.dst + p * limb_stride + off) = make_uint4(w[0], w[1], w[2], w[3]);
        }
    }
}

// ------------------------------------------------------------------------------------------------
// the GEMM
// ------------------------------------------------------------------------------------------------
template <typename T>
struct TcParams {
    const uint8_t *A_lo[2], *A_hi[2], *B_lo[2], *B_hi[2];  // tiled limb planes per party
    int64_t a_stride_lo, a_stride_hi, b_stride_lo, b_stride_hi;  // bytes between limb planes
    int nkb_lo, nkb_hi;                                          // K blocks in each half
    int kb_per_split;
    int64_t M, N;
    int nparty;
    int party_base;    // party of blockIdx.z % nparty == 0 (split deployment: the local party)
    int mode;          // 0 plain store, 1 Beaver (+Z_i, trunc), 2 dealer (Z1 = acc - Z0), 3 atomic partial
    T *C[2];
    const T *Z[2];
    int trunc;
    T *partial;        // mode 3: nparty x M x N
    int debug;         // experiments only (PSML_TC_DEBUG): 1 = skip pass-H stores, 2 = skip pass-L stores
};

// Epilogue chunk: thread `lane` holds 16 consecutive columns of row row0 + lane (the TMEM 32x32b
// fragment).  Transpose through a per-warp smem tile (32 x 17 words, padded) so that each store /
// read-modify-write instruction covers two 128-byte row segments instead of 32 scattered words.
// phase 0: v = low part (or the whole result in single-pass kernels); phase 1: v = high part.
template <typename T>
__device__ __forceinline__ void epi_chunk(T *st, const T v[16], int lane, int64_t row0, int64_t col0,
                                          const TcParams<T> &P, int party, int phase, bool two_pass) {
#pragma unroll
    for (int j = 0; j < 16; ++j) st[lane * 17 + j] = v[j];
    __syncwarp();
    const int c = lane & 15, rs = lane >> 4;
    const int64_t col = col0 + c;
#pragma unroll 4
    for (int r = 0; r < 16; ++r) {
        const int rl = 2 * r + rs;
        const int64_t row = row0 + rl;
        if (row >= P.M || col >= P.N) continue;
        const T x = st[rl * 17 + c];
        const int64_t o = row * P.N + col;
        if (P.mode == 3) {
            T *dst = P.partial + (int64_t)(party - P.party_base) * P.M * P.N + o;
            if (sizeof(T) == 8) atomicAdd((unsigned long long *)dst, (unsigned long long)x);
            else atomicAdd((unsigned int *)dst, (unsigned int)x);
            continue;
        }
        T *C = P.C[P.mode == 2 ? 0 : party];
        if (two_pass && phase == 0) { C[o] = x; continue; }
        const T acc = two_pass ? (T)(C[o] + x) : x;
        switch (P.mode) {
        case 0: C[o] = acc; break;
        case 1: C[o] = trunc_share<T>(acc + P.Z[party][o], party, P.trunc); break;
        default: C[o] = acc - P.Z[0][o]; break;
        }
    }
    __syncwarp();
}

#ifndef TC_B_MULTICAST
#define TC_B_MULTICAST 1
#endif
// MC = 2: the two CTAs of a (1, 2, 1) cluster (row blocks rb, rb + 1 of the same column block)
// share the B tile: each bulk-copies half of its limb planes to BOTH CTAs (TMA multicast), so the
// L2 -> SM traffic per block is A + B/2 instead of A + B (l = 32 at 4096^3 is L2-bandwidth bound:
// 4.3 GB of limb planes in 0.57 ms); each stage is freed only when both CTAs' MMAs retired it.
template <typename T, int L, int BN, int STAGES, int MC>
__global__ void __launch_bounds__(128, (STAGES * L * (BM * BK + BN * BK) <= 110 * 1024) ? 2 : 1)
    tc_ring_gemm_kernel(const TcParams<T> P) {
    extern __shared__ __align__(1024) uint8_t smem[];
    constexpr int A_BYTES = BM * BK, B_BYTES = BN * BK;
    // TMEM columns: L shift accumulators of BN columns (a power of two >= 32; 256 lets two CTAs
    // share an SM, one's epilogue overlapping the other's main loop)
    constexpr uint32_t TCOLS = L * BN <= 32 ? 32 : L * BN <= 64 ? 64 : L * BN <= 128 ? 128 : L * BN <= 256 ? 256 : 512;
    constexpr int STAGE_BYTES = L * (A_BYTES + B_BYTES);
    uint64_t *full = (uint64_t *)(smem + STAGES * STAGE_BYTES);
    uint64_t *empty = full + STAGES;
    uint64_t *accum = empty + STAGES;
    uint32_t *tmem_slot = (uint32_t *)(accum + 1);

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int party = P.party_base + blockIdx.z % P.nparty, split = blockIdx.z / P.nparty;
    const int nb = blockIdx.x, rb = blockIdx.y;
    const int nkb = P.nkb_lo + P.nkb_hi;
    const int kb0 = split * P.kb_per_split;
    const int kb1 = min(kb0 + P.kb_per_split, nkb);

    if (threadIdx.x == 0) {
        for (int s = 0; s < STAGES; ++s) {
            mbar_init(smem_u32(&full[s]), 1);
            mbar_init(smem_u32(&empty[s]), MC);
        }
        mbar_init(smem_u32(accum), 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 2) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)), "n"(TCOLS));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    tc_fence_before();
    if (MC > 1) cluster_sync_all();   // the peer's barriers exist before any multicast completes on them
    else __syncthreads();
    tc_fence_after();
    const uint32_t tmem = *tmem_slot;
    const uint32_t crank = MC > 1 ? cluster_rank() : 0;

    if (warp == 0 && lane == 0) {
        // ---------------- TMA producer ----------------
        int stage = 0;
        uint32_t phase = 0;
        for (int kb = kb0; kb < kb1; ++kb) {
            mbar_wait(smem_u32(&empty[stage]), phase ^ 1);
            const uint32_t fb = smem_u32(&full[stage]);
            mbar_expect_tx(fb, STAGE_BYTES);
            const bool lo = kb < P.nkb_lo;
            const int kk = lo ? kb : kb - P.nkb_lo;
            const int nk = lo ? P.nkb_lo : P.nkb_hi;
            const uint8_t *a = (lo ? P.A_lo[party] : P.A_hi[party]) + ((int64_t)rb * nk + kk) * A_BYTES;
            const uint8_t *b = (lo ? P.B_lo[party] : P.B_hi[party]) + ((int64_t)nb * nk + kk) * B_BYTES;
            const int64_t as = lo ? P.a_stride_lo : P.a_stride_hi, bs = lo ? P.b_stride_lo : P.b_stride_hi;
            uint8_t *sa = smem + stage * STAGE_BYTES, *sb = sa + L * A_BYTES;
#pragma unroll
            for (int p = 0; p < L; ++p) bulk_g2s(smem_u32(sa + p * A_BYTES), a + p * as, A_BYTES, fb);
            if (MC > 1) {
#pragma unroll
                for (int q = 0; q < L; ++q)
                    if (q % MC == (int)crank) bulk_g2s_mc(smem_u32(sb + q * B_BYTES), b + q * bs, B_BYTES, fb, (1u << MC) - 1);
            } else {
#pragma unroll
                for (int q = 0; q < L; ++q) bulk_g2s(smem_u32(sb + q * B_BYTES), b + q * bs, B_BYTES, fb);
            }
            if (++stage == STAGES) { stage = 0; phase ^= 1; }
        }
    } else if (warp == 1 && lane == 0) {
        // ---------------- MMA issuer: the l/8 (l/8 + 1) / 2 surviving limb pairs ----------------
        int stage = 0;
        uint32_t phase = 0;
        for (int kb = kb0; kb < kb1; ++kb) {
            mbar_wait(smem_u32(&full[stage]), phase);
            tc_fence_after();
            const uint32_t sa = smem_u32(smem + stage * STAGE_BYTES), sb = sa + L * A_BYTES;
            // the B planes q0, q0 + 1 of A limb p lie back to back in the canonical layout (plane
            // stride = BN / 8 row groups x SBO): ONE N = 2 BN operand into the adjacent shift
            // accumulators S_{p+q0}, S_{p+q0+1} -- 6 MMAs per block instead of 10 at l = 32, A read
            // 6 times instead of 10
            constexpr int GQ = 256 / BN;
#pragma unroll
            for (int p = 0; p < L; ++p) {
                const uint64_t ad = smem_desc(sa + p * A_BYTES, 128, 256);
#pragma unroll
                for (int q0 = 0; q0 < L - p; q0 += GQ) {
                    const int nq = (L - p - q0) < GQ ? (L - p - q0) : GQ;
                    const uint64_t bd = smem_desc(sb + q0 * B_BYTES, 128, 256);
                    tc_mma_i8(tmem + (uint32_t)((p + q0) * BN), ad, bd, idesc_i8(BM, nq * BN),
                              (kb > kb0 || p > 0) ? 1u : 0u);
                }
            }
            if (MC > 1) tc_commit_mc(smem_u32(&empty[stage]), (1u << MC) - 1);   // both CTAs' copies of the stage
            else tc_commit(smem_u32(&empty[stage]));   // frees the smem stage once these MMAs retire
            if (++stage == STAGES) { stage = 0; phase ^= 1; }
        }
        tc_commit(smem_u32(accum));               // all accumulators final
    }
    __syncwarp();

    // ---------------- epilogue: sum_s S_s 2^{8s} mod 2^l, + Z, trunc, store ----------------
    mbar_wait(smem_u32(accum), 0);
    tc_fence_after();
    const int64_t row0 = (int64_t)rb * BM + warp * 32;
    const uint32_t lane_base = tmem + ((uint32_t)(warp * 32) << 16);
    T *st = (T *)smem + warp * 32 * 17;   // pipeline smem is idle now: reuse it for staging
#pragma unroll 1
    for (int j0 = 0; j0 < BN; j0 += 16) {
        T acc[16];
#pragma unroll
        for (int j = 0; j < 16; ++j) acc[j] = 0;
#pragma unroll
        for (int s = 0; s < L; ++s) {
            uint32_t r[16];
            tmem_ld16(lane_base + (uint32_t)(s * BN + j0), r);
#pragma unroll
            for (int j = 0; j < 16; ++j) acc[j] += (T)r[j] << (8 * s);
        }
        epi_chunk<T>(st, acc, lane, row0, (int64_t)nb * BN + j0, P, party, 0, false);
    }
    tc_fence_before();
    if (MC > 1) cluster_sync_all();   // no CTA leaves while its peer's multicast / commits may still target it
    else __syncthreads();
    if (warp == 2) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "n"(TCOLS));
}

// ------------------------------------------------------------------------------------------------
// l = 64, v4: v2 with the passes reversed and the high half kept ON CHIP.
//   pass H first (shifts 4..7, 26 limb pairs): the epilogue warps fold the 4 accumulators into
//   high = sum S_s 2^{8(s-4)} mod 2^32 and park it in shared memory (128 x 128 x 4 B = 64 KB);
//   pass L (shifts 0..3, 10 limb pairs): the epilogue forms low + high 2^32 and stores C once.
// v2 staged the 64-bit pass-L partial through HBM (store + reload): measured 9-12% of the kernel.
// The 128 KB pipeline region is re-partitioned between passes: 2 x 64 KB stages in pass H
// (8 limbs of A and B per 32-byte K block), 4 x 32 KB stages in pass L (4 limbs each).
// ------------------------------------------------------------------------------------------------
__global__ void __launch_bounds__(192, 1) tc_ring_gemm64_v4(const TcParams<uint64_t> P) {
    using T = uint64_t;
    constexpr int BN = 128, L = 8;
    constexpr int A_BYTES = BM * BK, B_BYTES = BN * BK;
    constexpr int REGION = 2 * L * (A_BYTES + B_BYTES);               // 128 KB
    constexpr int SH_BYTES = L * (A_BYTES + B_BYTES), SL_BYTES = 4 * (A_BYTES + B_BYTES);
    constexpr uint32_t IDESC = idesc_i8(BM, BN);
    extern __shared__ __align__(1024) uint8_t smem[];
    uint32_t *hi_buf = (uint32_t *)(smem + REGION);                   // [col][row]
    uint64_t *bars = (uint64_t *)(smem + REGION + BM * BN * 4);
    uint64_t *fullH = bars, *emptyH = bars + 2, *fullL = bars + 4, *emptyL = bars + 8;
    uint64_t *accf = bars + 12, *acce = bars + 13;
    uint32_t *tmem_slot = (uint32_t *)(bars + 14);

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int party = P.party_base + blockIdx.z % P.nparty, split = blockIdx.z / P.nparty;
    const int nb = blockIdx.x, rb = blockIdx.y;
    const int nkb = P.nkb_lo + P.nkb_hi;
    const int kb0 = split * P.kb_per_split;
    const int kb1 = min(kb0 + P.kb_per_split, nkb);

    if (threadIdx.x == 0) {
        for (int s = 0; s < 2; ++s) { mbar_init(smem_u32(&fullH[s]), 1); mbar_init(smem_u32(&emptyH[s]), 1); }
        for (int s = 0; s < 4; ++s) { mbar_init(smem_u32(&fullL[s]), 1); mbar_init(smem_u32(&emptyL[s]), 1); }
        mbar_init(smem_u32(accf), 1);
        mbar_init(smem_u32(acce), 128);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 2) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(tmem_slot)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = *tmem_slot;

    auto tile_src = [&](int kb, const uint8_t *&a, const uint8_t *&b, int64_t &as, int64_t &bs) {
        const bool lo = kb < P.nkb_lo;
        const int kk = lo ? kb : kb - P.nkb_lo;
        const int nk = lo ? P.nkb_lo : P.nkb_hi;
        a = (lo ? P.A_lo[party] : P.A_hi[party]) + ((int64_t)rb * nk + kk) * A_BYTES;
        b = (lo ? P.B_lo[party] : P.B_hi[party]) + ((int64_t)nb * nk + kk) * B_BYTES;
        as = lo ? P.a_stride_lo : P.a_stride_hi;
        bs = lo ? P.b_stride_lo : P.b_stride_hi;
    };

    if (warp == 0) {
        if (lane == 0) {
            // ---------------- producer: pass H (2 x 64 KB), then pass L (4 x 32 KB) ----------------
            int st = 0;
            uint32_t ph = 0;
            for (int kb = kb0; kb < kb1; ++kb) {
                mbar_wait(smem_u32(&emptyH[st]), ph ^ 1);
                const uint32_t fb = smem_u32(&fullH[st]);
                mbar_expect_tx(fb, (uint32_t)SH_BYTES);
                const uint8_t *a, *b;
                int64_t as, bs;
                tile_src(kb, a, b, as, bs);
                uint8_t *sa = smem + st * SH_BYTES, *sb = sa + L * A_BYTES;
                for (int q = 0; q < L; ++q) bulk_g2s(smem_u32(sa + q * A_BYTES), a + q * as, A_BYTES, fb);
                for (int q = 0; q < L; ++q) bulk_g2s(smem_u32(sb + q * B_BYTES), b + q * bs, B_BYTES, fb);
                if (++st == 2) { st = 0; ph ^= 1; }
            }
            for (int i = 0; i < 2; ++i) {   // both pass-H slots consumed before re-partitioning
                mbar_wait(smem_u32(&emptyH[st]), ph ^ 1);
                if (++st == 2) { st = 0; ph ^= 1; }
            }
            st = 0;
            ph = 0;
            for (int kb = kb0; kb < kb1; ++kb) {
                mbar_wait(smem_u32(&emptyL[st]), ph ^ 1);
                const uint32_t fb = smem_u32(&fullL[st]);
                mbar_expect_tx(fb, (uint32_t)SL_BYTES);
                const uint8_t *a, *b;
                int64_t as, bs;
                tile_src(kb, a, b, as, bs);
                uint8_t *sa = smem + st * SL_BYTES, *sb = sa + 4 * A_BYTES;
                for (int q = 0; q < 4; ++q) bulk_g2s(smem_u32(sa + q * A_BYTES), a + q * as, A_BYTES, fb);
                for (int q = 0; q < 4; ++q) bulk_g2s(smem_u32(sb + q * B_BYTES), b + q * bs, B_BYTES, fb);
                if (++st == 4) { st = 0; ph ^= 1; }
            }
        }
    } else if (warp == 1) {
        if (lane == 0) {
            // ---------------- MMA issuer ----------------
            int st = 0;
            uint32_t ph = 0;
            for (int kb = kb0; kb < kb1; ++kb) {   // pass H: shifts 4..7
                mbar_wait(smem_u32(&fullH[st]), ph);
                tc_fence_after();
                const uint32_t sa = smem_u32(smem + st * SH_BYTES), sb = sa + L * A_BYTES;
#pragma unroll
                for (int p = 0; p < 8; ++p) {
                    const uint64_t ad = smem_desc(sa + p * A_BYTES, 128, 256);
#pragma unroll
                    for (int q = (p < 4 ? 4 - p : 0); q < 8 - p; ++q)
                        tc_mma_i8(tmem + (uint32_t)((p + q - 4) * BN), ad, smem_desc(sb + q * B_BYTES, 128, 256), IDESC,
                                  (kb > kb0 || p > 0) ? 1u : 0u);
                }
                tc_commit(smem_u32(&emptyH[st]));
                if (++st == 2) { st = 0; ph ^= 1; }
            }
            tc_commit(smem_u32(accf));
            mbar_wait(smem_u32(acce), 0);           // high half parked in smem, TMEM free
            tc_fence_after();
            st = 0;
            ph = 0;
            for (int kb = kb0; kb < kb1; ++kb) {   // pass L: shifts 0..3
                mbar_wait(smem_u32(&fullL[st]), ph);
                tc_fence_after();
                const uint32_t sa = smem_u32(smem + st * SL_BYTES), sb = sa + 4 * A_BYTES;
#pragma unroll
                for (int p = 0; p < 4; ++p) {
                    const uint64_t ad = smem_desc(sa + p * A_BYTES, 128, 256);
#pragma unroll
                    for (int q = 0; q < 4 - p; ++q)
                        tc_mma_i8(tmem + (uint32_t)((p + q) * BN), ad, smem_desc(sb + q * B_BYTES, 128, 256), IDESC,
                                  (kb > kb0 || p > 0) ? 1u : 0u);
                }
                tc_commit(smem_u32(&emptyL[st]));
                if (++st == 4) { st = 0; ph ^= 1; }
            }
            tc_commit(smem_u32(accf));
        }
    } else {
        // ---------------- epilogue warps 2..5 ----------------
        const int quarter = warp & 3;
        const int rl = quarter * 32 + lane;                 // row within the tile
        const int64_t row = (int64_t)rb * BM + rl;
        const uint32_t lane_base = tmem + ((uint32_t)(quarter * 32) << 16);
        const int64_t col0 = (int64_t)nb * BN;
        mbar_wait(smem_u32(accf), 0);
        tc_fence_after();
#pragma unroll 1
        for (int j0 = 0; j0 < BN; j0 += 16) {
            uint32_t hi[16];
#pragma unroll
            for (int j = 0; j < 16; ++j) hi[j] = 0;
#pragma unroll
            for (int s = 0; s < 4; ++s) {
                uint32_t r[16];
                tmem_ld16(lane_base + (uint32_t)(s * BN + j0), r);
#pragma unroll
                for (int j = 0; j < 16; ++j) hi[j] += r[j] << (8 * s);
            }
#pragma unroll
            for (int j = 0; j < 16; ++j) hi_buf[(j0 + j) * BM + rl] = hi[j];
        }
        tc_fence_before();
        mbar_arrive(smem_u32(acce));
        mbar_wait(smem_u32(accf), 1);
        tc_fence_after();
#pragma unroll 1
        for (int j0 = 0; j0 < BN; j0 += 16) {
            T acc[16];
#pragma unroll
            for (int j = 0; j < 16; ++j) acc[j] = (T)hi_buf[(j0 + j) * BM + rl] << 32;
#pragma unroll
            for (int s = 0; s < 4; ++s) {
                uint32_t r[16];
                tmem_ld16(lane_base + (uint32_t)(s * BN + j0), r);
#pragma unroll
                for (int j = 0; j < 16; ++j) acc[j] += (T)r[j] << (8 * s);
            }
            if (row < P.M && !(P.debug & 1)) {
#pragma unroll
                for (int j = 0; j < 16; ++j) {
                    const int64_t col = col0 + j0 + j;
                    if (col >= P.N) break;
                    const int64_t o = row * P.N + col;
                    switch (P.mode) {
                    case 0: P.C[party][o] = acc[j]; break;
                    case 1: P.C[party][o] = trunc_share<T>(acc[j] + P.Z[party][o], party, P.trunc); break;
                    case 2: P.C[0][o] = acc[j] - P.Z[0][o]; break;
                    default: atomicAdd((unsigned long long *)(P.partial + (int64_t)(party - P.party_base) * P.M * P.N + o), acc[j]);
                    }
                }
            }
        }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 2) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem));
}

constexpr size_t smem_v4_bytes() { return (size_t)2 * 8 * (BM * BK + 128 * BK) + (size_t)BM * 128 * 4 + 16 * 8; }

template <typename T>
__global__ void tc_finalize_kernel(const TcParams<T> P, int mode) {
    const int64_t total = P.M * P.N * P.nparty;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
        const int slot = (int)(i / (P.M * P.N));
        const int party = P.party_base + slot;
        const int64_t o = i - (int64_t)slot * P.M * P.N;
        const T acc = P.partial[i];
        if (mode == 0) P.C[party][o] = acc;
        else if (mode == 1) P.C[party][o] = trunc_share<T>(acc + P.Z[party][o], party, P.trunc);
        else P.C[0][o] = acc - P.Z[0][o];
    }
}

// ------------------------------------------------------------------------------------------------
// host side
// ------------------------------------------------------------------------------------------------
template <int l> struct Cfg;
// APAD: row padding of the A operand (l = 64 runs on CTA pairs: 256 rows per pair).
template <> struct Cfg<64> { using T = uint64_t; static constexpr int L = 8, BN = 128, STAGES = 3, APAD = 128; static constexpr int MAX_KB = 16384 / BK; };
#ifndef TC32_BN
#define TC32_BN 64
#endif
// l = 32: BN = 64 with 4 stages (98 KB, 256 TMEM columns) runs two CTAs per SM, one's epilogue
// beside the other's main loop (same box, + B multicast: 4096^3 0.578 -> 0.550 ms, 2048^3 0.118 ->
// 0.108 ms, 8192^3 4.04 -> 4.10 ms; BN = 128 without multicast 0.575 / 0.118 / 4.23 ms)
template <> struct Cfg<32> { using T = uint32_t; static constexpr int L = 4, BN = TC32_BN, STAGES = TC32_BN == 64 ? 4 : 6, APAD = 128; static constexpr int MAX_KB = 1 << 30; };

template <int l>
constexpr size_t smem_bytes() {
    return (size_t)Cfg<l>::STAGES * Cfg<l>::L * (BM * BK + Cfg<l>::BN * BK) + 256;
}

static inline int64_t rup(int64_t x, int64_t m) { return (x + m - 1) / m * m; }

// bytes of one tiled operand (all limbs); A operands (rt == BM) are padded to APAD rows
template <int l>
static int64_t tiled_bytes(int64_t rows, int64_t k, int rt) {
    const int pad = rt == BM ? Cfg<l>::APAD : rt;
    return (int64_t)Cfg<l>::L * rup(rows, pad) * rup(k, BK);
}

template <int l>
static SplitJob make_job(const void *s0, const void *s1, const void *s2, uint8_t *dst, int64_t rows, int64_t k,
                         int rt, int btype) {
    SplitJob j;
    const int pad = rt == BM ? Cfg<l>::APAD : rt;
    j.s0 = s0; j.s1 = s1; j.s2 = s2; j.dst = dst;
    j.rows = rows; j.kcols = k; j.rows_pad = rup(rows, pad); j.k_pad = rup(k, BK); j.rt = rt; j.btype = btype;
    return j;
}

template <int l>
static psml_status launch_split(const SplitJobs &jobs, cudaStream_t s) {
    int64_t units = 0;
    for (int i = 0; i < jobs.count; ++i) units = std::max(units, jobs.j[i].rows_pad * (jobs.j[i].k_pad / 16));
    dim3 grid((unsigned)grid_for(units, 256, 148 * 8), (unsigned)jobs.count);
    split_kernel<typename Cfg<l>::T, Cfg<l>::L><<<grid, 256, 0, s>>>(jobs);
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

// Picks split-K (fills the SMs, keeps each l = 64 pass exact) and launches GEMM (+ finalize).
template <int l>
static psml_status launch_gemm(TcParams<typename Cfg<l>::T> P, int64_t Mp, int64_t Np, typename Cfg<l>::T *partial,
                               int64_t partial_words, int sm_count, cudaStream_t s) {
    using T = typename Cfg<l>::T;
    constexpr int BN = Cfg<l>::BN;
    const int nkb = P.nkb_lo + P.nkb_hi;
    const int64_t tiles = (Mp / BM) * (Np / BN) * P.nparty;   // CTAs per split (pairs count 2)
    int splits = 1;
    if (tiles < sm_count)
        splits = (int)std::min<int64_t>((sm_count + tiles - 1) / tiles, std::max(1, nkb / PSML_TC_MINKB));
    splits = std::max(splits, (nkb + Cfg<l>::MAX_KB - 1) / Cfg<l>::MAX_KB);
    int kbs = (nkb + splits - 1) / splits;
    splits = (nkb + kbs - 1) / kbs;
    P.kb_per_split = kbs;
    P.debug = 0;
    const int final_mode = P.mode;
    if (splits > 1) {
        if (!partial || partial_words < P.M * P.N * P.nparty)
            return fail(PSML_ERR_NOMEM, "tcgen05 split-K workspace too small");
        P.partial = partial;
        P.mode = 3;
        PSML_CUDA_TRY(cudaMemsetAsync(partial, 0, sizeof(T) * P.M * P.N * P.nparty, s));
    }
    dim3 grid((unsigned)(Np / BN), (unsigned)(Mp / BM), (unsigned)(P.nparty * splits));
    {
        ProfScope prof(PROF_TC, s, (double)P.M * P.N * (double)(P.nkb_lo + P.nkb_hi) * BK * P.nparty);
        if constexpr (l == 64) {
            {
                auto kern = tc_ring_gemm64_v4;
                static bool attr_set = false;
                if (!attr_set) {
                    PSML_CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_v4_bytes()));
                    attr_set = true;
                }
                kern<<<grid, 192, smem_v4_bytes(), s>>>(P);
            }
        } else {
            auto kern1 = tc_ring_gemm_kernel<T, Cfg<l>::L, BN, Cfg<l>::STAGES, 1>;
            auto kern2 = tc_ring_gemm_kernel<T, Cfg<l>::L, BN, Cfg<l>::STAGES, 2>;
            static bool attr_set = false;
            if (!attr_set) {
                PSML_CUDA_TRY(cudaFuncSetAttribute(kern1, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_bytes<l>()));
                PSML_CUDA_TRY(cudaFuncSetAttribute(kern2, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_bytes<l>()));
                attr_set = true;
            }
            if (TC_B_MULTICAST && (Mp / BM) % 2 == 0) {   // row-block pairs share B (TMA multicast)
                cudaLaunchConfig_t cfg = {};
                cfg.gridDim = grid;
                cfg.blockDim = dim3(128);
                cfg.dynamicSmemBytes = smem_bytes<l>();
                cfg.stream = s;
                cudaLaunchAttribute at[1];
                at[0].id = cudaLaunchAttributeClusterDimension;
                at[0].val.clusterDim.x = 1; at[0].val.clusterDim.y = 2; at[0].val.clusterDim.z = 1;
                cfg.attrs = at;
                cfg.numAttrs = 1;
                PSML_CUDA_TRY(cudaLaunchKernelEx(&cfg, kern2, P));
            } else {
                kern1<<<grid, 128, smem_bytes<l>(), s>>>(P);
            }
        }
        PSML_LAUNCH_CHECK();
    }
    if (splits > 1) {
        tc_finalize_kernel<T><<<grid_for(P.M * P.N * P.nparty, 256), 256, 0, s>>>(P, final_mode);
        PSML_LAUNCH_CHECK();
    }
    return PSML_OK;
}

template <int l>
static size_t plain_ws_bytes(int64_t M, int64_t K, int64_t N) {
    using T = typename Cfg<l>::T;
    return (size_t)(tiled_bytes<l>(M, K, BM) + tiled_bytes<l>(N, K, Cfg<l>::BN) + 256 + (int64_t)sizeof(T) * M * N);
}

template <int l>
static psml_status plain_gemm(const void *A, const void *A2, const void *B, const void *B2, int64_t M, int64_t K,
                              int64_t N, void *C, const void *Z0, void *ws, size_t ws_bytes, cudaStream_t s) {
    using T = typename Cfg<l>::T;
    constexpr int BN = Cfg<l>::BN;
    if (ws_bytes < plain_ws_bytes<l>(M, K, N)) return fail(PSML_ERR_NOMEM, "tcgen05 workspace too small");
    uint8_t *ta = (uint8_t *)ws, *tb = ta + tiled_bytes<l>(M, K, BM);
    T *partial = (T *)(((uintptr_t)(tb + tiled_bytes<l>(N, K, BN)) + 255) & ~(uintptr_t)255);
    SplitJobs jobs;
    jobs.j[0] = make_job<l>(A, A2, nullptr, ta, M, K, BM, 0);
    jobs.j[1] = make_job<l>(B, B2, nullptr, tb, N, K, BN, 1);
    jobs.count = 2;
    {
        ProfScope prof(PROF_TC, s, 0.0);
        PSML_TRY(launch_split<l>(jobs, s));
    }
    TcParams<T> P{};
    P.A_lo[0] = P.A_lo[1] = ta; P.A_hi[0] = P.A_hi[1] = ta;
    P.B_lo[0] = P.B_lo[1] = tb; P.B_hi[0] = P.B_hi[1] = tb;
    P.a_stride_lo = P.a_stride_hi = jobs.j[0].rows_pad * jobs.j[0].k_pad;
    P.b_stride_lo = P.b_stride_hi = jobs.j[1].rows_pad * jobs.j[1].k_pad;
    P.nkb_lo = (int)(jobs.j[0].k_pad / BK); P.nkb_hi = 0;
    P.M = M; P.N = N; P.nparty = 1;
    P.mode = Z0 ? 2 : 0;
    P.C[0] = P.C[1] = (T *)C;
    P.Z[0] = P.Z[1] = (const T *)Z0;
    return launch_gemm<l>(P, jobs.j[0].rows_pad, jobs.j[1].rows_pad, partial, M * N, current_sm_count(), s);
}

}  // namespace tc

bool tc_available() { return true; }

size_t tc_ring_gemm_ws_bytes(int l, int64_t M, int64_t K, int64_t N) {
    return l == 64 ? tc::plain_ws_bytes<64>(M, K, N) : tc::plain_ws_bytes<32>(M, K, N);
}

psml_status tc_ring_gemm_plain(int l, const void *A, const void *B, int64_t M, int64_t K, int64_t N, void *C, void *ws,
                               size_t ws_bytes, cudaStream_t s) {
    if (l == 64) return tc::plain_gemm<64>(A, nullptr, B, nullptr, M, K, N, C, nullptr, ws, ws_bytes, s);
    return tc::plain_gemm<32>(A, nullptr, B, nullptr, M, K, N, C, nullptr, ws, ws_bytes, s);
}

// Dealer Z = (U0 + U1)(V0 + V1), Z1 = Z - Z0 (Z0 already generated), summing in the split.
psml_status tc_dealer_gemm(int l, const void *U0, const void *U1, const void *V0, const void *V1, int64_t M, int64_t K,
                           int64_t N, const void *Z0, void *Z1, void *ws, size_t ws_bytes, cudaStream_t s) {
    if (l == 64) return tc::plain_gemm<64>(U0, U1, V0, V1, M, K, N, Z1, Z0, ws, ws_bytes, s);
    return tc::plain_gemm<32>(U0, U1, V0, V1, M, K, N, Z1, Z0, ws, ws_bytes, s);
}

// ------------------------------------------------------------------------------------------------
// Beaver product on tensor cores.  After the mask round, the split round opens E and F and writes
// the limb planes of D'_0 = U_0, D'_1 = E + U_1, E (shared by both parties), F (shared), V_0, V_1;
// the GEMM walks K' = [lo half | hi half] = [D'_i | E] . [F ; V_i] (Eq. 8 in BJ form).
// ------------------------------------------------------------------------------------------------
template <typename T>
size_t tc_beaver_ws_bytes(int64_t M, int64_t K, int64_t N) {
    constexpr int l = 8 * (int)sizeof(T);
    const int64_t ta = tc::tiled_bytes<l>(M, K, tc::BM), tb = tc::tiled_bytes<l>(N, K, tc::Cfg<l>::BN);
    return (size_t)(sizeof(T) * (2 * M * K + 2 * K * N) + 3 * ta + 3 * tb + sizeof(T) * 2 * M * N + 4096);
}

template <typename T>
psml_status tc_beaver_matmul_ws(const T *const A[2], const T *const B[2], const T *const U[2], const T *const V[2],
                                const T *const Z[2], int64_t M, int64_t K, int64_t N, int flags, int trunc,
                                T *const C[2], void *ws, size_t ws_bytes, int sm_count, cudaStream_t s) {
    constexpr int l = 8 * (int)sizeof(T);
    using Cf = tc::Cfg<l>;
    if (tc_seg_small(l, M, 2 * K, N, 2, sm_count))   // small products: one open pass + the in-kernel split kernel
        return tc_seg_beaver<T>(A, B, U, V, Z, M, K, N, flags, trunc, C, ws, ws_bytes, s, sm_count);
    if (ws_bytes < tc_beaver_ws_bytes<T>(M, K, N)) return fail(PSML_ERR_NOMEM, "tcgen05 Beaver workspace too small");
    uint8_t *w = (uint8_t *)ws;
    auto carve = [&](size_t bytes) { uint8_t *p = w; w += (bytes + 255) & ~(size_t)255; return p; };
    T *mE0 = (T *)carve(sizeof(T) * M * K), *mE1 = (T *)carve(sizeof(T) * M * K);
    T *mF0 = (T *)carve(sizeof(T) * K * N), *mF1 = (T *)carve(sizeof(T) * K * N);
    const int64_t ta = tc::tiled_bytes<l>(M, K, tc::BM), tb = tc::tiled_bytes<l>(N, K, Cf::BN);
    uint8_t *tD0 = carve(ta), *tD1 = carve(ta), *tE = carve(ta), *tF = carve(tb), *tV0 = carve(tb), *tV1 = carve(tb);
    T *partial = (T *)carve(sizeof(T) * 2 * M * N);
    // round 1: masking (Eq. 4) -> messages
    const int tA = (flags & PSML_TRANS_A) ? 1 : 0, tB = (flags & PSML_TRANS_B) ? 1 : 0;
    MaskJobs<T> mj;
    mj.j[0] = {A[0], U[0], mE0, M, K, tA};
    mj.j[1] = {A[1], U[1], mE1, M, K, tA};
    mj.j[2] = {B[0], V[0], mF0, K, N, tB};
    mj.j[3] = {B[1], V[1], mF1, K, N, tB};
    mj.count = 4;
    const int64_t maxt = std::max(((M + 31) / 32) * ((K + 31) / 32), ((K + 31) / 32) * ((N + 31) / 32));
    {
        ProfScope prof(PROF_MASK, s, 3.0 * sizeof(T) * 2 * (M * K + K * N));
        mask_kernel<T><<<dim3((unsigned)std::min<int64_t>(maxt, 148 * 8), 1, 4), dim3(32, 8), 0, s>>>(mj);
        PSML_LAUNCH_CHECK();
    }
    // round 2a: open (Eq. 5) fused with the limb split
    tc::SplitJobs sj;
    sj.j[0] = tc::make_job<l>(U[0], nullptr, nullptr, tD0, M, K, tc::BM, 0);
    sj.j[1] = tc::make_job<l>(mE0, mE1, U[1], tD1, M, K, tc::BM, 0);
    sj.j[2] = tc::make_job<l>(mE0, mE1, nullptr, tE, M, K, tc::BM, 0);
    sj.j[3] = tc::make_job<l>(mF0, mF1, nullptr, tF, N, K, Cf::BN, 1);
    sj.j[4] = tc::make_job<l>(V[0], nullptr, nullptr, tV0, N, K, Cf::BN, 1);
    sj.j[5] = tc::make_job<l>(V[1], nullptr, nullptr, tV1, N, K, Cf::BN, 1);
    sj.count = 6;
    {
        ProfScope prof(PROF_TC, s, 0.0);
        PSML_TRY(tc::launch_split<l>(sj, s));
    }
    // round 2b: the ring GEMM with the Beaver epilogue
    tc::TcParams<T> P{};
    P.A_lo[0] = tD0; P.A_lo[1] = tD1; P.A_hi[0] = P.A_hi[1] = tE;
    P.B_lo[0] = P.B_lo[1] = tF; P.B_hi[0] = tV0; P.B_hi[1] = tV1;
    P.a_stride_lo = P.a_stride_hi = sj.j[0].rows_pad * sj.j[0].k_pad;
    P.b_stride_lo = P.b_stride_hi = sj.j[3].rows_pad * sj.j[3].k_pad;
    P.nkb_lo = P.nkb_hi = (int)(sj.j[0].k_pad / tc::BK);
    P.M = M; P.N = N; P.nparty = 2; P.mode = 1; P.trunc = trunc;
    P.C[0] = C[0]; P.C[1] = C[1]; P.Z[0] = Z[0]; P.Z[1] = Z[1];
    return tc::launch_gemm<l>(P, sj.j[0].rows_pad, sj.j[3].rows_pad, partial, 2 * M * N, sm_count, s);
}

template <typename T>
psml_status tc_beaver_matmul(Ctx *c, const T *const A[2], const T *const B[2], const T *const U[2], const T *const V[2],
                             const T *const Z[2], int64_t M, int64_t K, int64_t N, int flags, int trunc, T *const C[2],
                             cudaStream_t s) {
    PSML_TRY(c->ensure_ws(tc_beaver_ws_bytes<T>(M, K, N)));
    return tc_beaver_matmul_ws<T>(A, B, U, V, Z, M, K, N, flags, trunc, C, c->ws, c->ws_bytes, c->sm_count, s);
}

// Split deployment, round 2 for ONE party: the split round opens E = E_send + E_recv and
// F = F_send + F_recv while writing the limb planes of D'_i (= U_0, or E + U_1), E, F and V_i.
template <int l>
static psml_status open_matmul_one(Ctx *c, int party, const void *Es, const void *Er, const void *Fs, const void *Fr,
                                   const void *U, const void *V, const void *Z, int64_t M, int64_t K, int64_t N,
                                   int trunc, void *C, cudaStream_t s) {
    using Cf = tc::Cfg<l>;
    using T = typename Cf::T;
    const int64_t ta = tc::tiled_bytes<l>(M, K, tc::BM), tb = tc::tiled_bytes<l>(N, K, Cf::BN);
    const size_t need = (size_t)(2 * ta + 2 * tb + sizeof(T) * M * N + 2048);
    PSML_TRY(c->ensure_ws(need));
    uint8_t *w = (uint8_t *)c->ws;
    auto carve = [&](size_t bytes) { uint8_t *p = w; w += (bytes + 255) & ~(size_t)255; return p; };
    uint8_t *tD = carve(ta), *tE = carve(ta), *tF = carve(tb), *tV = carve(tb);
    T *partial = (T *)carve(sizeof(T) * M * N);
    tc::SplitJobs sj;
    sj.j[0] = party == 0 ? tc::make_job<l>(U, nullptr, nullptr, tD, M, K, tc::BM, 0)
                         : tc::make_job<l>(Es, Er, U, tD, M, K, tc::BM, 0);
    sj.j[1] = tc::make_job<l>(Es, Er, nullptr, tE, M, K, tc::BM, 0);
    sj.j[2] = tc::make_job<l>(Fs, Fr, nullptr, tF, N, K, Cf::BN, 1);
    sj.j[3] = tc::make_job<l>(V, nullptr, nullptr, tV, N, K, Cf::BN, 1);
    sj.count = 4;
    {
        ProfScope prof(PROF_TC, s, 0.0);
        PSML_TRY(tc::launch_split<l>(sj, s));
    }
    tc::TcParams<T> P{};
    P.A_lo[0] = P.A_lo[1] = tD; P.A_hi[0] = P.A_hi[1] = tE;
    P.B_lo[0] = P.B_lo[1] = tF; P.B_hi[0] = P.B_hi[1] = tV;
    P.a_stride_lo = P.a_stride_hi = sj.j[0].rows_pad * sj.j[0].k_pad;
    P.b_stride_lo = P.b_stride_hi = sj.j[2].rows_pad * sj.j[2].k_pad;
    P.nkb_lo = P.nkb_hi = (int)(sj.j[0].k_pad / tc::BK);
    P.M = M; P.N = N; P.nparty = 1; P.party_base = party; P.mode = 1; P.trunc = trunc;
    P.C[0] = P.C[1] = (T *)C; P.Z[0] = P.Z[1] = (const T *)Z;
    return tc::launch_gemm<l>(P, sj.j[0].rows_pad, sj.j[2].rows_pad, partial, M * N, c->sm_count, s);
}

psml_status tc_open_matmul_one(Ctx *c, int l, int party, const void *Es, const void *Er, const void *Fs,
                               const void *Fr, const void *U, const void *V, const void *Z, int64_t M, int64_t K,
                               int64_t N, int trunc, void *C, cudaStream_t s) {
    if (l == 64) return open_matmul_one<64>(c, party, Es, Er, Fs, Fr, U, V, Z, M, K, N, trunc, C, s);
    return open_matmul_one<32>(c, party, Es, Er, Fs, Fr, U, V, Z, M, K, N, trunc, C, s);
}

template size_t tc_beaver_ws_bytes<uint64_t>(int64_t, int64_t, int64_t);
template size_t tc_beaver_ws_bytes<uint32_t>(int64_t, int64_t, int64_t);
template psml_status tc_beaver_matmul_ws<uint64_t>(const uint64_t *const[2], const uint64_t *const[2],
                                                   const uint64_t *const[2], const uint64_t *const[2],
                                                   const uint64_t *const[2], int64_t, int64_t, int64_t, int, int,
                                                   uint64_t *const[2], void *, size_t, int, cudaStream_t);

template psml_status tc_beaver_matmul<uint64_t>(Ctx *, const uint64_t *const[2], const uint64_t *const[2],
                                                const uint64_t *const[2], const uint64_t *const[2],
                                                const uint64_t *const[2], int64_t, int64_t, int64_t, int, int,
                                                uint64_t *const[2], cudaStream_t);
template psml_status tc_beaver_matmul<uint32_t>(Ctx *, const uint32_t *const[2], const uint32_t *const[2],
                                                const uint32_t *const[2], const uint32_t *const[2],
                                                const uint32_t *const[2], int64_t, int64_t, int64_t, int, int,
                                                uint32_t *const[2], cudaStream_t);

}  // namespace psml
