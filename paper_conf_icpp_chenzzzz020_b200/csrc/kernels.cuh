// kernels.cuh -- elementwise / protocol-round kernels of libpsml (co-resident pair engine).
//
// Round structure: every protocol round is ONE kernel that (1) opens the
// previous round's messages -- reading party 0's and party 1's masked words from their send
// buffers in HBM (Eq. 5), (2) does the local computation of both parties, and (3)
// writes this round's masked messages.  A thread owns one element for both parties, so each
// opened word is read once and all accesses are coalesced 8-byte (l=64) / 4-byte (l=32) words.
#pragma once
#include "common.cuh"

namespace psml {

template <typename T> struct Pair { T *p[2]; };
template <typename T> struct CPair { const T *p[2]; };

// ---------------------------------------------------------------------------------------------
// PRG fill / encode / decode / share / reconstruct  (client side)
// ---------------------------------------------------------------------------------------------
// One thread per ChaCha20 block; OP = 0: out = prg; 1: out = x - prg (share: x1) and x0 = prg.
template <typename T, int OP>
__global__ void prg_kernel(PrgKey key, uint64_t offset, int64_t n, T *__restrict__ out,
                           const T *__restrict__ x, T *__restrict__ out2) {
    constexpr int PB = PerBlock<T>::value;
    key = live_key(key);
    const uint64_t first_blk = offset / PB;
    const uint64_t last_blk = (offset + (uint64_t)n - 1) / PB;
    for (uint64_t b = first_blk + (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; b <= last_blk;
         b += (uint64_t)gridDim.x * blockDim.x) {
        uint32_t w[16];
        chacha20_block(key, (uint32_t)b, w);
#pragma unroll
        for (int j = 0; j < PB; ++j) {
            uint64_t e = b * PB + j;
            if (e < offset || e >= offset + (uint64_t)n) continue;
            T v = sizeof(T) == 8 ? (T)(((uint64_t)w[2 * j + 1] << 32) | w[2 * j]) : (T)w[j];
            int64_t i = (int64_t)(e - offset);
            if (OP == 0) out[i] = v;
            else { out[i] = v; out2[i] = x[i] - v; }
        }
    }
}

// Client encode + share in one pass: v = encode(x) (R3), x0 = PRG, x1 = v - x0.
template <typename T>
__global__ void encode_share_kernel(PrgKey key, int64_t n, int f, const double *__restrict__ x, T *__restrict__ out0,
                                    T *__restrict__ out1) {
    constexpr int PB = PerBlock<T>::value;
    key = live_key(key);
    const uint64_t last_blk = ((uint64_t)n - 1) / PB;
    for (uint64_t b = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; b <= last_blk; b += (uint64_t)gridDim.x * blockDim.x) {
        uint32_t w[16];
        chacha20_block(key, (uint32_t)b, w);
#pragma unroll
        for (int j = 0; j < PB; ++j) {
            const uint64_t e = b * PB + j;
            if (e >= (uint64_t)n) continue;
            const T r = sizeof(T) == 8 ? (T)(((uint64_t)w[2 * j + 1] << 32) | w[2 * j]) : (T)w[j];
            const T v = (T)(unsigned long long)__double2ll_rn(ldexp(x[e], f));
            out0[e] = r;
            out1[e] = v - r;
        }
    }
}

// Same, with the plaintext given as bytes: x = q / den (pixels, den = 255) or, for den = 0, the
// one-hot row of class index q[e / classes] (x = 1 at column q, else 0).
template <typename T>
__global__ void encode_share_u8_kernel(PrgKey key, int64_t n, int f, const uint8_t *__restrict__ q, double den,
                                       int64_t classes, T *__restrict__ out0, T *__restrict__ out1) {
    constexpr int PB = PerBlock<T>::value;
    key = live_key(key);
    const uint64_t last_blk = ((uint64_t)n - 1) / PB;
    for (uint64_t b = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; b <= last_blk; b += (uint64_t)gridDim.x * blockDim.x) {
        uint32_t w[16];
        chacha20_block(key, (uint32_t)b, w);
#pragma unroll
        for (int j = 0; j < PB; ++j) {
            const uint64_t e = b * PB + j;
            if (e >= (uint64_t)n) continue;
            const T r = sizeof(T) == 8 ? (T)(((uint64_t)w[2 * j + 1] << 32) | w[2 * j]) : (T)w[j];
            double x;
            if (den > 0.0) x = (double)q[e] / den;
            else x = (int64_t)q[e / (uint64_t)classes] == (int64_t)(e % (uint64_t)classes) ? 1.0 : 0.0;
            const T v = (T)(unsigned long long)__double2ll_rn(ldexp(x, f));
            out0[e] = r;
            out1[e] = v - r;
        }
    }
}

template <typename T>
__global__ void encode_kernel(const double *__restrict__ x, int64_t n, int f, T *__restrict__ v) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        long long r = __double2ll_rn(ldexp(x[i], f));   // round half to even (R3)
        v[i] = (T)(unsigned long long)r;
    }
}

template <typename T>
__global__ void decode_kernel(const T *__restrict__ v, int64_t n, int f, double *__restrict__ x) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        double s = sizeof(T) == 8 ? (double)(long long)(uint64_t)v[i] : (double)(int)(uint32_t)v[i];
        x[i] = ldexp(s, -f);
    }
}

template <typename T>
__global__ void add_kernel(const T *__restrict__ a, const T *__restrict__ b, int64_t n, T *__restrict__ c) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        c[i] = a[i] + b[i];
}

template <typename T>
__global__ void truncate_kernel(T *__restrict__ x, int64_t n, int party, int d) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        x[i] = trunc_share<T>(x[i], party, d);
}

// ---------------------------------------------------------------------------------------------
// dealer kernels (offline; Eqs. 2-3, Fig. 4; R4, R9)
// ---------------------------------------------------------------------------------------------
// U0,U1 (or V0,V1) streams + their sum (written to `sum`, used as the GEMM operand for Z).
template <typename T>
__global__ void dealer_pair_kernel(PrgKey k0, PrgKey k1, int64_t n, T *__restrict__ o0,
                                   T *__restrict__ o1, T *__restrict__ sum) {
    constexpr int PB = PerBlock<T>::value;
    k0 = live_key(k0);
    k1 = live_key(k1);
    const int64_t nblk = (n + PB - 1) / PB;
    for (int64_t b = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; b < nblk; b += (int64_t)gridDim.x * blockDim.x) {
        uint32_t w0[16], w1[16];
        chacha20_block(k0, (uint32_t)b, w0);
        chacha20_block(k1, (uint32_t)b, w1);
#pragma unroll
        for (int j = 0; j < PB; ++j) {
            int64_t e = b * PB + j;
            if (e >= n) break;
            T v0 = sizeof(T) == 8 ? (T)(((uint64_t)w0[2 * j + 1] << 32) | w0[2 * j]) : (T)w0[j];
            T v1 = sizeof(T) == 8 ? (T)(((uint64_t)w1[2 * j + 1] << 32) | w1[2 * j]) : (T)w1[j];
            o0[e] = v0; o1[e] = v1;
            if (sum) sum[e] = v0 + v1;
        }
    }
}

template <typename T>
__device__ __forceinline__ T word_of(const uint32_t *w, int j) {
    return sizeof(T) == 8 ? (T)(((uint64_t)w[2 * j + 1] << 32) | w[2 * j]) : (T)w[j];
}

// Hadamard triplet: Z_1 = (U0+U1)(V0+V1) - Z0, elementwise.
template <typename T>
__global__ void hadamard_triplet_kernel(PrgKey ku0, PrgKey ku1, PrgKey kv0, PrgKey kv1, PrgKey kz0,
                                        int64_t n, Pair<T> U, Pair<T> V, Pair<T> Z) {
    constexpr int PB = PerBlock<T>::value;
    ku0 = live_key(ku0); ku1 = live_key(ku1); kv0 = live_key(kv0); kv1 = live_key(kv1); kz0 = live_key(kz0);
    const int64_t nblk = (n + PB - 1) / PB;
    for (int64_t b = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; b < nblk; b += (int64_t)gridDim.x * blockDim.x) {
        uint32_t a0[16], a1[16], c0[16], c1[16], z[16];
        chacha20_block(ku0, (uint32_t)b, a0);
        chacha20_block(ku1, (uint32_t)b, a1);
        chacha20_block(kv0, (uint32_t)b, c0);
        chacha20_block(kv1, (uint32_t)b, c1);
        chacha20_block(kz0, (uint32_t)b, z);
#pragma unroll
        for (int j = 0; j < PB; ++j) {
            int64_t e = b * PB + j;
            if (e >= n) break;
            T u0 = word_of<T>(a0, j), u1 = word_of<T>(a1, j), v0 = word_of<T>(c0, j), v1 = word_of<T>(c1, j);
            T z0 = word_of<T>(z, j);
            U.p[0][e] = u0; U.p[1][e] = u1; V.p[0][e] = v0; V.p[1][e] = v1;
            Z.p[0][e] = z0; Z.p[1][e] = (T)((u0 + u1) * (v0 + v1)) - z0;
        }
    }
}

// MSB material of the reduced prefix (R27): blockIdx.y = group g (0 .. 2) or 3 for the
// daBit.  Group g's a / b / c words are masked to its gate bits (msb_group_mask).
__host__ __device__ inline uint64_t low_bits(int w) { return w >= 64 ? ~(uint64_t)0 : (((uint64_t)1 << w) - 1); }
__host__ __device__ inline uint64_t msb_group_mask(int l, int g) {
    if (g == 0) return low_bits(l - 1);                    // round 0: bits 0 .. l-2
    if (g == 1) return low_bits(l - 1) & ~(uint64_t)1;     // level 1: bits 1 .. l-2
    uint64_t m = 0;                                        // levels 2..: fields of l/2, l/4, ... bits
    int off = 0;
    for (int w = l / 2; w >= 2; w /= 2) {
        m |= (low_bits(w) & ~(uint64_t)1) << off;
        off += w;
    }
    return m;
}
constexpr int MSB_WORDS = 11;   // 3 groups x (a, b, c) + daBit (r^B, r^A), per element and party

template <typename T>
__global__ void msb_dealer_kernel(const DealSeeds S, uint64_t call_id, int64_t n, int L, T *__restrict__ m0,
                                  T *__restrict__ m1, const uint32_t *step) {
    constexpr int PB = PerBlock<uint64_t>::value;
    constexpr int l = 8 * (int)sizeof(T);
    (void)L;
    if (step) {
        const uint64_t st = *step;
        call_id = (call_id & ~(0xFFFFFFFFull << 24)) | (st << 24);
    }
    const int g = blockIdx.y;
    const int64_t nblk = (n + PB - 1) / PB;
    const uint64_t gm = g < 3 ? msb_group_mask(l, g) : 0;
    for (int64_t b = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; b < nblk; b += (int64_t)gridDim.x * blockDim.x) {
        if (g < 3) {
            uint32_t wa0[16], wa1[16], wb0[16], wb1[16], wc0[16];
            chacha20_block(dkey(S, tag4('a', '0', g), call_id), (uint32_t)b, wa0);
            chacha20_block(dkey(S, tag4('a', '1', g), call_id), (uint32_t)b, wa1);
            chacha20_block(dkey(S, tag4('b', '0', g), call_id), (uint32_t)b, wb0);
            chacha20_block(dkey(S, tag4('b', '1', g), call_id), (uint32_t)b, wb1);
            chacha20_block(dkey(S, tag4('c', '0', g), call_id), (uint32_t)b, wc0);
            T *base0 = m0 + (int64_t)g * 3 * n, *base1 = m1 + (int64_t)g * 3 * n;
#pragma unroll
            for (int j = 0; j < PB; ++j) {
                int64_t e = b * PB + j;
                if (e >= n) break;
                const uint64_t a0 = word_of<uint64_t>(wa0, j) & gm, a1 = word_of<uint64_t>(wa1, j) & gm;
                const uint64_t b0 = word_of<uint64_t>(wb0, j) & gm, b1 = word_of<uint64_t>(wb1, j) & gm;
                const uint64_t c0 = word_of<uint64_t>(wc0, j) & gm;
                base0[e] = (T)a0; base0[n + e] = (T)b0; base0[2 * n + e] = (T)c0;
                base1[e] = (T)a1; base1[n + e] = (T)b1; base1[2 * n + e] = (T)(((a0 ^ a1) & (b0 ^ b1)) ^ c0);
            }
        }
    }
    if (g == 3) {   // daBit: r^B_i = PRG(R, i) & 1 (l-bit stream), r^A_0 = PRG(R, A), r^A_1 = r - r^A_0
        constexpr int PBT = PerBlock<T>::value;
        const int64_t nbt = (n + PBT - 1) / PBT;
        for (int64_t b = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; b < nbt; b += (int64_t)gridDim.x * blockDim.x) {
            uint32_t w0[16], w1[16], wa[16];
            chacha20_block(dkey(S, TAG_R0, call_id), (uint32_t)b, w0);
            chacha20_block(dkey(S, TAG_R1, call_id), (uint32_t)b, w1);
            chacha20_block(dkey(S, TAG_RA, call_id), (uint32_t)b, wa);
            const int64_t off = (int64_t)9 * n;
#pragma unroll
            for (int j = 0; j < PBT; ++j) {
                int64_t e = b * PBT + j;
                if (e >= n) break;
                T r0 = word_of<T>(w0, j) & 1, r1 = word_of<T>(w1, j) & 1, ra0 = word_of<T>(wa, j);
                m0[off + e] = r0; m1[off + e] = r1;
                m0[off + n + e] = ra0; m1[off + n + e] = (T)(r0 ^ r1) - ra0;
            }
        }
    }
}

// ---------------------------------------------------------------------------------------------
// Beaver masking (Eq. 4): up to 4 jobs (E_0, E_1, F_0, F_1), each dst = op(src) - mask, with an
// optional transpose of src staged through a 32x33 shared tile.
// ---------------------------------------------------------------------------------------------
template <typename T>
struct MaskJob {
    const T *src;   // rows x cols in op layout (or cols x rows if trans)
    const T *mask;  // rows x cols
    T *dst;         // rows x cols
    int64_t rows, cols;
    int trans;
};
template <typename T> struct MaskJobs { MaskJob<T> j[4]; int count; };

template <typename T>
__global__ void mask_kernel(MaskJobs<T> jobs) {
    __shared__ T tile[32][33];
    const MaskJob<T> J = jobs.j[blockIdx.z];
    const int64_t tiles_c = (J.cols + 31) / 32;
    const int64_t tiles = ((J.rows + 31) / 32) * tiles_c;
    for (int64_t t = blockIdx.x; t < tiles; t += gridDim.x) {
        const int64_t r0 = (t / tiles_c) * 32, c0 = (t % tiles_c) * 32;
        if (J.trans) {
            // src stored cols x rows: read coalesced along rows, write coalesced along cols
            __syncthreads();
            for (int i = threadIdx.y; i < 32; i += blockDim.y) {
                int64_t sc = c0 + i, sr = r0 + threadIdx.x;
                tile[i][threadIdx.x] = (sc < J.cols && sr < J.rows) ? J.src[sc * J.rows + sr] : (T)0;
            }
            __syncthreads();
            for (int i = threadIdx.y; i < 32; i += blockDim.y) {
                int64_t r = r0 + i, c = c0 + threadIdx.x;
                if (r < J.rows && c < J.cols) J.dst[r * J.cols + c] = tile[threadIdx.x][i] - J.mask[r * J.cols + c];
            }
        } else {
            for (int i = threadIdx.y; i < 32; i += blockDim.y) {
                int64_t r = r0 + i, c = c0 + threadIdx.x;
                if (r < J.rows && c < J.cols) {
                    int64_t o = r * J.cols + c;
                    J.dst[o] = J.src[o] - J.mask[o];
                }
            }
        }
    }
}

// ---------------------------------------------------------------------------------------------
// Beaver Hadamard: round 1 masks, round 2 opens and combines (BJ form), optional truncation.
// ---------------------------------------------------------------------------------------------
template <typename T>
__global__ void hadamard_mask_kernel(CPair<T> A, CPair<T> B, CPair<T> U, CPair<T> V, int64_t n,
                                     Pair<T> mE, Pair<T> mF, int only = -1) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
#pragma unroll
        for (int p = 0; p < 2; ++p) {
            if (only >= 0 && p != only) continue;
            mE.p[p][i] = A.p[p][i] - U.p[p][i];
            mF.p[p][i] = B.p[p][i] - V.p[p][i];
        }
    }
}

// ---------------------------------------------------------------------------------------------
// Secure MSB chain (R9): Kogge-Stone carry on boolean shares, one kernel per round.
// Input modes: 0 = x as given (n elements); 1 = Eq. 9 pair [z + h ; z - h] over z of n/2
// elements (party 0 adds the public +-h, h = 2^(f-1)).
// State per party: G, P words.  Messages per party: up to 4 words (e, f of two ANDs).
// ---------------------------------------------------------------------------------------------
template <typename T>
struct MsbArgs {
    CPair<T> x;        // input shares (n, or n/2 in mode 1)
    CPair<T> mat;      // dealer material
    Pair<T> G, P;      // state, n words per party
    Pair<T> msg;       // 4 n words per party
    int64_t n;
    int mode;
    T half;            // 2^(f-1) for mode 1
    int L, l;
    // -1: co-resident (both parties).  0 / 1: split deployment -- this process is party `only`;
    // msg.p[only] is its send buffer and msg.p[1 - only] the peer's received words (same layout).
    int only = -1;
};
#define PSML_PARTY_SKIP(a, p) \
    if ((a).only >= 0 && (p) != (a).only) continue;

template <typename T>
__device__ __forceinline__ T msb_input(const MsbArgs<T> &a, int p, int64_t e) {
    if (a.mode == 0) return a.x.p[p][e];
    const int64_t h = a.n >> 1;
    if (e < h) return a.x.p[p][e] + (p == 0 ? a.half : (T)0);
    return a.x.p[p][e - h] - (p == 0 ? a.half : (T)0);
}

template <typename T>
__device__ __forceinline__ const T *mat_ptr(const MsbArgs<T> &a, int p, int g, int w) {
    return a.mat.p[p] + ((int64_t)g * 3 + w) * a.n;
}

// ---- the reduced Kogge-Stone prefix (R27) ---------------------------------------------
// Bit gather of positions start, start + 2, ... of v into the low bits (start 0: even, 1: odd).
__device__ __forceinline__ uint64_t compact_bits(uint64_t x, int start) {
    x = (x >> start) & 0x5555555555555555ull;
    x = (x | (x >> 1)) & 0x3333333333333333ull;
    x = (x | (x >> 2)) & 0x0F0F0F0F0F0F0F0Full;
    x = (x | (x >> 4)) & 0x00FF00FF00FF00FFull;
    x = (x | (x >> 8)) & 0x0000FFFF0000FFFFull;
    x = (x | (x >> 16)) & 0x00000000FFFFFFFFull;
    return x;
}
// Level j = 1 .. L of an l-bit prefix: word width w = l >> (j - 1); material group (1 for j = 1,
// else 2 at field offset l - 2w); gate masks of the G and P ANDs.
struct MsbLevel {
    int w, group, off;
    uint64_t MG, MP;
};
__device__ __forceinline__ MsbLevel msb_level(int l, int j) {
    MsbLevel v;
    v.w = l >> (j - 1);
    if (j == 1) {   // even positions 2 .. l-2, both gates
        v.group = 1; v.off = 0;
        v.MG = v.MP = 0x5555555555555555ull & low_bits(l - 1) & ~(uint64_t)1;
    } else {        // odd positions (P: >= 3) of the compacted w-bit word
        v.group = 2; v.off = l - 2 * v.w;
        v.MG = 0xAAAAAAAAAAAAAAAAull & low_bits(v.w);
        v.MP = v.MG & ~(uint64_t)2;
    }
    return v;
}
// unpack a group word into the level's G-gate and P-gate material (P stored shifted down by one)
__device__ __forceinline__ void msb_unpack(const MsbLevel &v, uint64_t word, uint64_t &gpart, uint64_t &ppart) {
    const uint64_t f = (word >> v.off) & low_bits(v.w);
    gpart = f & v.MG;
    ppart = (f << 1) & v.MP;
}
// one restricted boolean Beaver AND for party p: z_p = (p ? e&f : 0) ^ (e & b_p) ^ (a_p & f) ^ c_p
__device__ __forceinline__ uint64_t and_z(int p, uint64_t e, uint64_t f, uint64_t a, uint64_t b, uint64_t c) {
    const uint64_t r = (e & b) ^ (a & f) ^ c;
    return p == 1 ? (r ^ (e & f)) : r;
}

// ---- per-element round bodies (one protocol round each) -----------------------------------------
// Round 1: mask AND 0 (G = X0 & X1 on bits 0 .. l-2) with X = (x0, 0), Y = (0, x1).
template <typename T>
__device__ __forceinline__ void msb_round0_body(const MsbArgs<T> &a, int64_t e) {
    const uint64_t M0 = low_bits(a.l - 1);
#pragma unroll
    for (int p = 0; p < 2; ++p) {
        PSML_PARTY_SKIP(a, p)
        const uint64_t x = (uint64_t)msb_input(a, p, e);
        const uint64_t X = p == 0 ? x : 0, Y = p == 1 ? x : 0;
        a.msg.p[p][e] = (T)((X ^ (uint64_t)mat_ptr(a, p, 0, 0)[e]) & M0);
        a.msg.p[p][a.n + e] = (T)((Y ^ (uint64_t)mat_ptr(a, p, 0, 1)[e]) & M0);
    }
}

// open the AND of level jp (0 = round 0) from message words 0, 1: G / P of both parties, compacted
template <typename T>
__device__ __forceinline__ void msb_open_level(const MsbArgs<T> &a, int64_t e, int jp, uint64_t G[2], uint64_t P[2]) {
    const uint64_t E = (uint64_t)a.msg.p[0][e] ^ (uint64_t)a.msg.p[1][e];
    const uint64_t Fo = (uint64_t)a.msg.p[0][a.n + e] ^ (uint64_t)a.msg.p[1][a.n + e];
    if (jp == 0) {
#pragma unroll
        for (int p = 0; p < 2; ++p) {
            PSML_PARTY_SKIP(a, p)
            G[p] = and_z(p, E, Fo, mat_ptr(a, p, 0, 0)[e], mat_ptr(a, p, 0, 1)[e], mat_ptr(a, p, 0, 2)[e]);
            P[p] = (uint64_t)msb_input(a, p, e);
        }
        return;
    }
    const MsbLevel v = msb_level(a.l, jp);
    uint64_t eG, eP, fG, fP;
    msb_unpack(MsbLevel{v.w, v.group, 0, v.MG, v.MP}, E, eG, eP);   // messages are packed at offset 0
    msb_unpack(MsbLevel{v.w, v.group, 0, v.MG, v.MP}, Fo, fG, fP);
#pragma unroll
    for (int p = 0; p < 2; ++p) {
        PSML_PARTY_SKIP(a, p)
        uint64_t aG, aP, bG, bP, cG, cP;
        msb_unpack(v, mat_ptr(a, p, v.group, 0)[e], aG, aP);
        msb_unpack(v, mat_ptr(a, p, v.group, 1)[e], bG, bP);
        msb_unpack(v, mat_ptr(a, p, v.group, 2)[e], cG, cP);
        const uint64_t zG = and_z(p, eG, fG, aG, bG, cG), zP = and_z(p, eP, fP, aP, bP, cP);
        const int start = jp == 1 ? 0 : 1;
        G[p] = compact_bits((uint64_t)a.G.p[p][e] ^ zG, start);
        P[p] = compact_bits(zP, start);
    }
}

// Round j+1 (j = 1..L): open level j-1's AND, mask level j's G and P ANDs (one packed word each).
template <typename T>
__device__ __forceinline__ void msb_level_body(const MsbArgs<T> &a, int j, int64_t e) {
    uint64_t G[2] = {0, 0}, P[2] = {0, 0};
    msb_open_level(a, e, j - 1, G, P);
    const MsbLevel v = msb_level(a.l, j);
#pragma unroll
    for (int p = 0; p < 2; ++p) {
        PSML_PARTY_SKIP(a, p)
        uint64_t aG, aP, bG, bP;
        msb_unpack(v, mat_ptr(a, p, v.group, 0)[e], aG, aP);
        msb_unpack(v, mat_ptr(a, p, v.group, 1)[e], bG, bP);
        const uint64_t eG = (P[p] ^ aG) & v.MG, fG = ((G[p] << 1) ^ bG) & v.MG;
        const uint64_t eP = (P[p] ^ aP) & v.MP, fP = ((P[p] << 1) ^ bP) & v.MP;
        a.msg.p[p][e] = (T)(eG | (eP >> 1));
        a.msg.p[p][a.n + e] = (T)(fG | (fP >> 1));
        a.G.p[p][e] = (T)G[p];
        a.P.p[p][e] = (T)P[p];
    }
}

// Round L+2: open the last level's AND, msb_i = x_i[l-1] ^ G_i[l-2] (bit 0 of the compacted G);
// emit the B2A message c_i.
template <typename T>
__device__ __forceinline__ void msb_final_body(const MsbArgs<T> &a, const Pair<T> &msbB, int64_t e) {
    const int64_t off = (int64_t)9 * a.n;
    uint64_t G[2] = {0, 0}, P[2] = {0, 0};
    msb_open_level(a, e, a.L, G, P);
#pragma unroll
    for (int p = 0; p < 2; ++p) {
        PSML_PARTY_SKIP(a, p)
        const T x = msb_input(a, p, e);
        const T b = ((x >> (a.l - 1)) & 1) ^ (T)(G[p] & 1);
        if (msbB.p[p]) msbB.p[p][e] = b;
        a.msg.p[p][e] = b ^ a.mat.p[p][off + e];   // c_i = msb_i ^ rB_i
    }
}

// Round L+3: open c, [msb]^A; then either store msbA (what = 0) or, for ReLU/Eq. 9 (what = 1),
// form drelu_i = [i==0] - msbA_i and mask the Hadamard x . drelu (messages mE, mF).
template <typename T>
__device__ __forceinline__ void msb_b2a_body(const MsbArgs<T> &a, const Pair<T> &msbA, const Pair<T> &drelu,
                                             const CPair<T> &U, const CPair<T> &V, const Pair<T> &mE,
                                             const Pair<T> &mF, int what, int64_t e) {
    const int64_t off = (int64_t)9 * a.n;
    const T c = a.msg.p[0][e] ^ a.msg.p[1][e];
    const T s = (T)1 - (T)2 * c;
#pragma unroll
    for (int p = 0; p < 2; ++p) {
        PSML_PARTY_SKIP(a, p)
        T m = (p == 0 ? c : (T)0) + s * a.mat.p[p][off + a.n + e];
        if (what == 0) {
            msbA.p[p][e] = m;
        } else {
            T d = (p == 0 ? (T)1 : (T)0) - m;
            if (drelu.p[p]) drelu.p[p][e] = d;
            mE.p[p][e] = msb_input(a, p, e) - U.p[p][e];
            mF.p[p][e] = d - V.p[p][e];
        }
    }
}

template <typename T>
__device__ __forceinline__ void hadamard_open_body(const CPair<T> &mE, const CPair<T> &mF, const CPair<T> &U,
                                                   const CPair<T> &V, const CPair<T> &Z, int trunc,
                                                   const Pair<T> &C, int64_t i, int only = -1) {
    const T e = mE.p[0][i] + mE.p[1][i], f = mF.p[0][i] + mF.p[1][i];
#pragma unroll
    for (int p = 0; p < 2; ++p) {
        if (only >= 0 && p != only) continue;
        T c = (T)p * e * f + e * V.p[p][i] + U.p[p][i] * f + Z.p[p][i];
        C.p[p][i] = trunc_share<T>(c, p, trunc);
    }
}

// Round L+4 for Eq. 9: open the Hadamard of 2n' elements, y_i = r_i[e] - r_i[e + n'].
template <typename T>
__device__ __forceinline__ void eq9_open_body(const CPair<T> &mE, const CPair<T> &mF, const CPair<T> &U,
                                              const CPair<T> &V, const CPair<T> &Z, int64_t nh, const Pair<T> &y,
                                              const CPair<T> &Ysub, const Pair<T> &delta, int64_t e,
                                              int only = -1) {
    const T e1 = mE.p[0][e] + mE.p[1][e], f1 = mF.p[0][e] + mF.p[1][e];
    const T e2 = mE.p[0][e + nh] + mE.p[1][e + nh], f2 = mF.p[0][e + nh] + mF.p[1][e + nh];
#pragma unroll
    for (int p = 0; p < 2; ++p) {
        if (only >= 0 && p != only) continue;
        T r1 = (T)p * e1 * f1 + e1 * V.p[p][e] + U.p[p][e] * f1 + Z.p[p][e];
        T r2 = (T)p * e2 * f2 + e2 * V.p[p][e + nh] + U.p[p][e + nh] * f2 + Z.p[p][e + nh];
        T out = r1 - r2;
        if (y.p[p]) y.p[p][e] = out;
        if (delta.p[p]) delta.p[p][e] = out - Ysub.p[p][e];
    }
}

#define PSML_GRID_LOOP(e, n) \
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < (n); e += (int64_t)gridDim.x * blockDim.x)

// ---- one kernel per round (the split-deployment structure; also the fallback) --------------------
template <typename T>
__global__ void msb_round0_kernel(MsbArgs<T> a) { PSML_GRID_LOOP(e, a.n) msb_round0_body(a, e); }

template <typename T>
__global__ void msb_level_kernel(MsbArgs<T> a, int j) { PSML_GRID_LOOP(e, a.n) msb_level_body(a, j, e); }

template <typename T>
__global__ void msb_final_kernel(MsbArgs<T> a, Pair<T> msbB) { PSML_GRID_LOOP(e, a.n) msb_final_body(a, msbB, e); }

template <typename T>
__global__ void msb_b2a_kernel(MsbArgs<T> a, Pair<T> msbA, Pair<T> drelu, CPair<T> U, CPair<T> V,
                               Pair<T> mE, Pair<T> mF, int what) {
    PSML_GRID_LOOP(e, a.n) msb_b2a_body(a, msbA, drelu, U, V, mE, mF, what, e);
}

template <typename T>
__global__ void hadamard_open_kernel(CPair<T> mE, CPair<T> mF, CPair<T> U, CPair<T> V, CPair<T> Z,
                                     int64_t n, int trunc, Pair<T> C, int only = -1) {
    PSML_GRID_LOOP(i, n) hadamard_open_body(mE, mF, U, V, Z, trunc, C, i, only);
}

template <typename T>
__global__ void eq9_open_kernel(CPair<T> mE, CPair<T> mF, CPair<T> U, CPair<T> V, CPair<T> Z,
                                int64_t nh, Pair<T> y, CPair<T> Ysub, Pair<T> delta, int only = -1) {
    PSML_GRID_LOOP(e, nh) eq9_open_body(mE, mF, U, V, Z, nh, y, Ysub, delta, e, only);
}

// ---- the whole chain in ONE launch, rounds in order per element ----------------------------------
// In the co-resident engine, round r+1 of element e only opens the two parties' round-r messages
// of the same element e.  One thread therefore runs element e through every round in protocol
// order -- each round still writes both parties' masked messages to their send buffers and the
// next round opens them from there -- so the chain costs one launch instead of one per round.
// (A split deployment exchanges the messages between rounds instead: msb_*_kernel per round.)
// Eq. 9 pairs element e with e + n/2 so its final opening stays thread-local.
// Opening of one consumer operand from a produced rows x cols matrix v (row-major, index e), used
// by the fused training step (fused.cuh): dst index di = e (trans = 0) or (e % cols) * rows +
// e / cols (the consumer reads v^T); E[di] = (v_0 - M_0[di]) + (v_1 - M_1[di]) and, for an A side,
// X1[di] = E[di] + M_1[di].
template <typename T>
struct Emit {
    const T *M[2];
    T *E, *X1;
    int64_t rows, cols;
    int trans;
};
template <typename T>
struct Emits {
    Emit<T> e[2];
    int n;
};
template <typename T>
__device__ __forceinline__ int64_t emit_index(const Emit<T> &em, int64_t e) {
    return em.trans ? (e % em.cols) * em.rows + e / em.cols : e;
}

template <typename T>
struct ChainOut {
    Pair<T> msbA, msbB, drelu, y, delta;
    CPair<T> U, V, Z, Ysub;
    Pair<T> mE, mF;
    int what;
    Emits<T> em;   // consumer opens of y (ReLU) / delta (Eq. 9); lane-pair kernel only
};

template <typename T>
__device__ __forceinline__ void msb_chain_element(const MsbArgs<T> &a, const ChainOut<T> &o, int64_t e) {
    msb_round0_body(a, e);
#pragma unroll 1
    for (int j = 1; j <= a.L; ++j) msb_level_body(a, j, e);
    msb_final_body(a, o.msbB, e);
    msb_b2a_body(a, o.msbA, o.drelu, o.U, o.V, o.mE, o.mF, o.what == 0 ? 0 : 1, e);
}

template <typename T>
__global__ void __launch_bounds__(256) msb_chain_fused_kernel(MsbArgs<T> a, ChainOut<T> o) {
    CPair<T> ce{{o.mE.p[0], o.mE.p[1]}}, cf{{o.mF.p[0], o.mF.p[1]}};
    if (o.what == 2) {
        const int64_t nh = a.n / 2;
        PSML_GRID_LOOP(e, nh) {
            msb_chain_element(a, o, e);
            msb_chain_element(a, o, e + nh);
            eq9_open_body(ce, cf, o.U, o.V, o.Z, nh, o.y, o.Ysub, o.delta, e);
        }
        return;
    }
    PSML_GRID_LOOP(e, a.n) {
        msb_chain_element(a, o, e);
        if (o.what == 1) hadamard_open_body(ce, cf, o.U, o.V, o.Z, 0, o.y, e);
    }
}

// ---- the whole chain in one launch, one LANE PER PARTY ------------------------------------------
// Lanes 2i and 2i+1 run the same element for party 0 and party 1.  Each round a lane computes its
// party's masked words and obtains the peer's words with a lane-pair shuffle -- the co-resident
// form of the opening (Eq. 5 / boolean e = x ^ a); the messages never touch memory (the
// per-round kernels, PSML_MSB_CHAIN=rounds, write them to the send buffers a split deployment
// exchanges).  G, P and all dealer material stay in registers.  MODE 0: msb, 1: ReLU,
// 2: Eq. 9 (lanes 0-15 run 8 elements of the first half [z + 1/2], lanes 16-31 the matching
// elements of the second half [z - 1/2]; the final difference is a shuffle by 16).
template <typename T>
__device__ __forceinline__ T peer_of(T v) {
    return (T)__shfl_xor_sync(0xffffffffu, (unsigned long long)v, 1);
}

#define SEL(pair) (p ? (pair).p[1] : (pair).p[0])
template <typename T, int MODE>
__global__ void __launch_bounds__(256) msb_chain_pair_kernel(MsbArgs<T> a, ChainOut<T> o) {
    pdl_trigger();
    constexpr int l = 8 * (int)sizeof(T);
    constexpr int L = sizeof(T) == 8 ? 6 : 5;
    const int lane = threadIdx.x & 31;
    const int p = lane & 1;
    const int64_t gtid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t n = a.n;
    int64_t e;
    bool valid, second = false;
    if (MODE == 2) {
        const int64_t nh = n >> 1;
        const int64_t base = (gtid >> 5) * 8 + ((lane >> 1) & 7);
        second = lane >= 16;
        valid = base < nh;
        e = valid ? (second ? base + nh : base) : 0;
    } else {
        e = gtid >> 1;
        valid = e < n;
        if (!valid) e = 0;
    }
    const T *mat = p ? a.mat.p[1] : a.mat.p[0];
    // Every load of the chain is data-independent: issue them all up front (one memory round trip
    // instead of one per protocol round -- the rounds' message stores would otherwise order them).
    // The dealer material (AND triplets, daBit, Hadamard triplet, the consumers' masks) was
    // written by a kernel that completed before any PDL predecessor of this one could start (the
    // previous graph's dealer, or a dealer launch without early trigger), so it is loaded BEFORE
    // griddepcontrol.wait, overlapping the predecessor's tail; only x depends on the predecessor.
    uint64_t mt[3][3];   // the reduced prefix's material (R27): 3 groups x (a, b, c)
#pragma unroll
    for (int g = 0; g < 3; ++g)
#pragma unroll
        for (int w = 0; w < 3; ++w) mt[g][w] = (uint64_t)mat[((int64_t)g * 3 + w) * n + e];
    const int64_t off = (int64_t)9 * n;
    const T rB = mat[off + e], rA = mat[off + n + e];
    T hu = 0, hv = 0, hz = 0, ysub = 0;
    if (MODE != 0) { hu = SEL(o.U)[e]; hv = SEL(o.V)[e]; hz = SEL(o.Z)[e]; }
    T emk[2] = {0, 0};
    int64_t edi[2] = {0, 0};
#pragma unroll
    for (int q = 0; q < 2; ++q)
        if (q < o.em.n && (MODE != 2 || !second)) {
            edi[q] = emit_index(o.em.e[q], e);
            emk[q] = o.em.e[q].M[p][edi[q]];
        }
    pdl_wait();
    const T *xin = p ? a.x.p[1] : a.x.p[0];
    const T half = p == 0 ? a.half : (T)0;
    const T x = a.mode == 0 ? xin[e] : (e < (n >> 1) ? xin[e] + half : xin[e - (n >> 1)] - half);
    if (MODE == 2 && !second && SEL(o.Ysub)) ysub = SEL(o.Ysub)[e];
    // consumer opens of this lane pair's value v (both parties: v here, the peer's by shuffle)
    auto emit = [&](T v, bool ok) {
#pragma unroll
        for (int q = 0; q < 2; ++q) {
            if (q >= o.em.n) break;
            const T part = v - emk[q];
            const T E = part + peer_of(part);
            if (ok) {
                if (p == 0) o.em.e[q].E[edi[q]] = E;
                else if (o.em.e[q].X1) o.em.e[q].X1[edi[q]] = E + emk[q];
            }
        }
    };
    // round 1: AND 0 on X = (x0, 0), Y = (0, x1), bits 0 .. l-2
    const uint64_t M0 = low_bits(l - 1), xw = (uint64_t)x;
    const uint64_t m0 = ((p == 0 ? xw : 0) ^ mt[0][0]) & M0, m1 = ((p == 1 ? xw : 0) ^ mt[0][1]) & M0;
    uint64_t G = and_z(p, m0 ^ peer_of(m0), m1 ^ peer_of(m1), mt[0][0], mt[0][1], mt[0][2]);
    uint64_t P = xw;
#pragma unroll
    for (int j = 1; j <= L; ++j) {   // one round per level: the packed G and P ANDs
        const MsbLevel v = msb_level(l, j);
        uint64_t aG, aP, bG, bP, cG, cP;
        msb_unpack(v, mt[v.group][0], aG, aP);
        msb_unpack(v, mt[v.group][1], bG, bP);
        msb_unpack(v, mt[v.group][2], cG, cP);
        const uint64_t eG = (P ^ aG) & v.MG, fG = ((G << 1) ^ bG) & v.MG;
        const uint64_t eP = (P ^ aP) & v.MP, fP = ((P << 1) ^ bP) & v.MP;
        const uint64_t me = eG | (eP >> 1), mf = fG | (fP >> 1);   // this party's two message words
        const uint64_t E = me ^ peer_of(me), Fo = mf ^ peer_of(mf);
        const uint64_t oG = E & v.MG, oP = (E << 1) & v.MP, qG = Fo & v.MG, qP = (Fo << 1) & v.MP;
        const uint64_t zG = and_z(p, oG, qG, aG, bG, cG), zP = and_z(p, oP, qP, aP, bP, cP);
        const int start = j == 1 ? 0 : 1;
        G = compact_bits(G ^ zG, start);
        P = compact_bits(zP, start);
    }
    const T bit = ((x >> (l - 1)) & 1) ^ (T)(G & 1);
    if (valid && SEL(o.msbB)) SEL(o.msbB)[e] = bit;
    const T cm = bit ^ rB;                    // B2A: c_i = msb_i ^ rB_i
    const T c = cm ^ peer_of(cm);
    const T mA = (p == 0 ? c : (T)0) + ((T)1 - (T)2 * c) * rA;
    if (MODE == 0) {
        if (valid) SEL(o.msbA)[e] = mA;
        return;
    }
    const T d = (p == 0 ? (T)1 : (T)0) - mA;  // DReLU share
    if (valid && SEL(o.drelu)) SEL(o.drelu)[e] = d;
    const T u = hu, v = hv;
    const T me = x - u, mf = d - v;           // Hadamard round: mask
    const T E = me + peer_of(me), F = mf + peer_of(mf);
    const T r = (T)p * E * F + E * v + u * F + hz;
    if (MODE == 1) {
        if (valid && SEL(o.y)) SEL(o.y)[e] = r;
        emit(r, valid);
        return;
    }
    const T r2 = (T)__shfl_xor_sync(0xffffffffu, (unsigned long long)r, 16);
    const T out = r - r2;                     // ReLU(z + 1/2) - ReLU(z - 1/2)
    const T dl = out - ysub;
    if (valid && !second) {
        if (SEL(o.y)) SEL(o.y)[e] = out;
        if (SEL(o.delta)) SEL(o.delta)[e] = dl;
    }
    emit(dl, valid && !second);
}

#undef SEL

// ---------------------------------------------------------------------------------------------
// training helpers
// ---------------------------------------------------------------------------------------------
template <typename T>
__global__ void sub_pair_kernel(CPair<T> a, CPair<T> b, int64_t n, Pair<T> c, int only = -1) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        if (only != 1) c.p[0][i] = a.p[0][i] - b.p[0][i];
        if (only != 0) c.p[1][i] = a.p[1][i] - b.p[1][i];
    }
}

// W^m_i -= trunc_i(g_i, s_grad) [+ trunc_i(W^m_i, wd): weight decay, SVM R24]; W_i = trunc_i(W^m_i, s_fwd)
// (R14, R21)
template <typename T>
__global__ void update_kernel(Pair<T> Wm, Pair<T> W, CPair<T> g, int64_t n, int s_grad, int s_fwd, int only = -1,
                              int wd = 0) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
#pragma unroll
        for (int p = 0; p < 2; ++p) {
            if (only >= 0 && p != only) continue;
            const T old = Wm.p[p][i];
            const T dec = wd ? trunc_share<T>(old, p, wd) : (T)0;
            T wm = old - (trunc_share<T>(g.p[p][i], p, s_grad) + dec);
            Wm.p[p][i] = wm;
            W.p[p][i] = trunc_share<T>(wm, p, s_fwd);
        }
    }
}

template <typename T>
__global__ void truncate_pair_kernel(CPair<T> src, Pair<T> dst, int64_t n, int d) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        dst.p[0][i] = trunc_share<T>(src.p[0][i], 0, d);
        dst.p[1][i] = trunc_share<T>(src.p[1][i], 1, d);
    }
}

}  // namespace psml
