/*
 * psml_oracle.c -- CPU ORACLE for the ParSecureML hot path.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may
 * load this library.  It shares no code, header, table or constant generator with the CUDA
 * path under paper_conf_icpp_chenzzzz020_b200/ and never includes anything from it.
 *
 * What it is: a plain, slow, obviously-correct simulation of BOTH parties of the two-party
 * Beaver-triplet protocol in the ring Z_{2^l} (values stored in uint64_t, reduced mod 2^l),
 * written in the paper's order and notation:
 *   PAPER.md L65-L78 (Sec. 2.2, Eqs. 1-6)  triplet multiplication, masking, opening, C_i
 *   PAPER.md L164-L176 (Sec. 4.2, Eqs. 7-8) one-GEMM form (only used as a cross-check)
 *   PAPER.md L178-L181 (Eq. 9)              piecewise-linear activation
 *   PAPER.md L215-L228 (Eqs. 10-12)          delta + CSR compressed transmission
 * plus the readings DESIGN.md lists where the paper is silent (ring, PRG, truncation, MSB
 * protocol: DESIGN.md "Readings" R1..R18).
 *
 * Every loop is the textbook definition: no blocking, no fusion, no reordering.  The only
 * concession to speed is `#pragma omp parallel for` over independent output rows/elements,
 * which does not change any arithmetic (ring addition is exact).
 *
 * Parity pins (tests/test_oracle_*.py, marked "not gpu"):
 *   chacha20 block      -> RFC 8439 Sec. 2.3.2 / 2.4.2 known-answer vectors
 *   ring matmul         -> Python big-int brute force (independent arithmetic)
 *   triplets / Beaver   -> closed forms Z0+Z1 = (U0+U1)(V0+V1), C0+C1 = A.B mod 2^l
 *   truncation          -> SecureML Thm. 1 bound + stochastic-rounding statistics
 *   MSB / ReLU / Eq. 9  -> exhaustive over all x in toy rings l = 8, 16 vs the sign bit
 *   CSR codec           -> round trip and the 75%-zeros format rule
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>

#define EXPORT __attribute__((visibility("default")))

static inline uint64_t ring_mask(int l) { return l >= 64 ? ~(uint64_t)0 : (((uint64_t)1 << l) - 1); }

/* ------------------------------------------------------------------------------------------ */
/* ChaCha20 block function, RFC 8439 Sec. 2.3 (R1: the PRG replacing MT19937 of       */
/* PAPER.md L246).                                                                            */
/* ------------------------------------------------------------------------------------------ */
static inline uint32_t rotl32(uint32_t v, int c) { return (v << c) | (v >> (32 - c)); }

#define QR(a, b, c, d)                 \
    a += b; d ^= a; d = rotl32(d, 16); \
    c += d; b ^= c; b = rotl32(b, 12); \
    a += b; d ^= a; d = rotl32(d, 8);  \
    c += d; b ^= c; b = rotl32(b, 7);

EXPORT void or_chacha20_block(const uint32_t key[8], uint32_t counter, const uint32_t nonce[3],
                              uint32_t out[16]) {
    uint32_t s[16], x[16];
    s[0] = 0x61707865u; s[1] = 0x3320646eu; s[2] = 0x79622d32u; s[3] = 0x6b206574u;
    for (int i = 0; i < 8; ++i) s[4 + i] = key[i];
    s[12] = counter;
    s[13] = nonce[0]; s[14] = nonce[1]; s[15] = nonce[2];
    for (int i = 0; i < 16; ++i) x[i] = s[i];
    for (int r = 0; r < 10; ++r) {
        QR(x[0], x[4], x[8], x[12]);
        QR(x[1], x[5], x[9], x[13]);
        QR(x[2], x[6], x[10], x[14]);
        QR(x[3], x[7], x[11], x[15]);
        QR(x[0], x[5], x[10], x[15]);
        QR(x[1], x[6], x[11], x[12]);
        QR(x[2], x[7], x[8], x[13]);
        QR(x[3], x[4], x[9], x[14]);
    }
    for (int i = 0; i < 16; ++i) out[i] = x[i] + s[i];
}

/*
 * PRG stream (R1): key = seed as 8 little-endian bytes || 24 zero bytes;
 * nonce = 4-byte role tag || 8-byte call id, little endian; block counter = element / per_block.
 * l > 32: element e = words (2j, 2j+1) of block e/8, j = e%8, little endian -> uint64.
 * l <= 32: element e = word e%16 of block e/16.  Result reduced mod 2^l.
 */
EXPORT void or_prg(int l, uint64_t seed, uint32_t tag, uint64_t id, uint64_t offset, int64_t n,
                   uint64_t *out) {
    uint32_t key[8] = {(uint32_t)seed, (uint32_t)(seed >> 32), 0, 0, 0, 0, 0, 0};
    uint32_t nonce[3] = {tag, (uint32_t)id, (uint32_t)(id >> 32)};
    uint64_t m = ring_mask(l);
    int per_block = l > 32 ? 8 : 16;
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) {
        uint64_t e = offset + (uint64_t)i;
        uint32_t blk[16];
        or_chacha20_block(key, (uint32_t)(e / per_block), nonce, blk);
        int j = (int)(e % per_block);
        uint64_t v = l > 32 ? ((uint64_t)blk[2 * j] | ((uint64_t)blk[2 * j + 1] << 32)) : blk[j];
        out[i] = v & m;
    }
}

/*
 * Dealer key separation (R23).  The dealer (the paper's client) holds the
 * dealer seed; party i holds only s_i = first word of PRG(dealer_seed, "KD", i) (R1 layout).  Every
 * material stream a party can produce itself is keyed by that party's seed (U0, V0, Z0, a0, b0, c0,
 * R0, RA, F0, FS, K0 -> s_0; U1, V1, a1, b1, R1, K1 -> s_1); streams only the dealer may know (the
 * FSS input mask "FR") keep the dealer seed.  The derived words (Z_1, c_1, r^A_1, FSS correction
 * words) need both seeds and are what the dealer ships (compressed distribution).
 */
EXPORT uint64_t or_party_seed(uint64_t dealer_seed, int party) {
    uint64_t v;
    or_prg(64, dealer_seed, 0x0000444Bu /* "KD" */, (uint64_t)party, 0, 1, &v);
    return v;
}

EXPORT uint64_t or_stream_seed(uint64_t dealer_seed, uint32_t tag) {
    int b0 = (int)(tag & 0xFF), b1 = (int)((tag >> 8) & 0xFF);
    if (b1 == '1') return or_party_seed(dealer_seed, 1);
    if (b1 == '0' || (b0 == 'R' && b1 == 'A') || (b0 == 'F' && b1 == 'S')) return or_party_seed(dealer_seed, 0);
    return dealer_seed;
}

/* or_prg for a dealer material stream: keyed by or_stream_seed. */
static void dprg(int l, uint64_t seed, uint32_t tag, uint64_t id, uint64_t offset, int64_t n, uint64_t *out) {
    or_prg(l, or_stream_seed(seed, tag), tag, id, offset, n, out);
}

/* ------------------------------------------------------------------------------------------ */
/* Fixed-point encoding (R3; SecureML fixed point, not in PAPER.md which is FP32,     */
/* L248/L260): v = round_half_even(x * 2^f) mod 2^l;  decode = signed(v) / 2^f.               */
/* ------------------------------------------------------------------------------------------ */
EXPORT void or_encode(int l, int f, const double *x, int64_t n, uint64_t *v) {
    uint64_t m = ring_mask(l);
    for (int64_t i = 0; i < n; ++i) {
        long long r = llrint(ldexp(x[i], f)); /* default FP env: round half to even */
        v[i] = (uint64_t)r & m;
    }
}

EXPORT void or_decode(int l, int f, const uint64_t *v, int64_t n, double *x) {
    uint64_t m = ring_mask(l);
    for (int64_t i = 0; i < n; ++i) {
        uint64_t u = v[i] & m;
        int64_t s;
        if (l < 64 && (u >> (l - 1)) & 1) s = (int64_t)(u - m - 1); /* u - 2^l */
        else s = (int64_t)u;
        x[i] = ldexp((double)s, -f);
    }
}

/* ------------------------------------------------------------------------------------------ */
/* Additive 2-party sharing, PAPER.md L65 ("randomly divide matrix A into A_0 and A_1") and    */
/* L238 (A_0 random, A_1 by subtraction).  x_0 = PRG(seed, "SH", stream), x_1 = x - x_0.       */
/* ------------------------------------------------------------------------------------------ */
#define TAG(a, b, c, d) ((uint32_t)(uint8_t)(a) | ((uint32_t)(uint8_t)(b) << 8) | \
                         ((uint32_t)(uint8_t)(c) << 16) | ((uint32_t)(uint8_t)(d) << 24))

EXPORT void or_share(int l, uint64_t seed, uint64_t stream, const uint64_t *x, int64_t n,
                     uint64_t *x0, uint64_t *x1) {
    uint64_t m = ring_mask(l);
    or_prg(l, seed, TAG('S', 'H', 0, 0), stream, 0, n, x0);
    for (int64_t i = 0; i < n; ++i) x1[i] = (x[i] - x0[i]) & m;
}

EXPORT void or_reconstruct(int l, const uint64_t *x0, const uint64_t *x1, int64_t n, uint64_t *x) {
    uint64_t m = ring_mask(l);
    for (int64_t i = 0; i < n; ++i) x[i] = (x0[i] + x1[i]) & m;
}

/* Plain ring matmul C = A (MxK) . B (KxN) mod 2^l, row-major, schoolbook triple loop. */
EXPORT void or_ring_matmul(int l, const uint64_t *A, const uint64_t *B, int64_t M, int64_t K,
                           int64_t N, uint64_t *C) {
    uint64_t m = ring_mask(l);
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < M; ++i) {
        for (int64_t j = 0; j < N; ++j) {
            uint64_t acc = 0;
            for (int64_t k = 0; k < K; ++k) acc += A[i * K + k] * B[k * N + j];
            C[i * N + j] = acc & m;
        }
    }
}

/* ------------------------------------------------------------------------------------------ */
/* Dealer (offline phase, Eqs. 2-3, Fig. 4): U, V random, Z = U x V,     */
/* split into shares.  Reading R4: U_0,U_1,V_0,V_1,Z_0 from PRG streams, Z_1 = U V - Z_0.      */
/* kind 0 = matrix triplet (U: MxK, V: KxN, Z: MxN); kind 1 = Hadamard (all n = M elements).   */
/* ------------------------------------------------------------------------------------------ */
EXPORT void or_triplet_gen(int l, uint64_t seed, uint64_t call_id, int64_t M, int64_t K, int64_t N,
                           uint64_t *U0, uint64_t *U1, uint64_t *V0, uint64_t *V1, uint64_t *Z0,
                           uint64_t *Z1) {
    uint64_t m = ring_mask(l);
    dprg(l, seed, TAG('U', '0', 0, 0), call_id, 0, M * K, U0);
    dprg(l, seed, TAG('U', '1', 0, 0), call_id, 0, M * K, U1);
    dprg(l, seed, TAG('V', '0', 0, 0), call_id, 0, K * N, V0);
    dprg(l, seed, TAG('V', '1', 0, 0), call_id, 0, K * N, V1);
    dprg(l, seed, TAG('Z', '0', 0, 0), call_id, 0, M * N, Z0);
    uint64_t *U = malloc(sizeof(uint64_t) * M * K), *V = malloc(sizeof(uint64_t) * K * N);
    uint64_t *Z = malloc(sizeof(uint64_t) * M * N);
    for (int64_t i = 0; i < M * K; ++i) U[i] = (U0[i] + U1[i]) & m;   /* Eq. 3 */
    for (int64_t i = 0; i < K * N; ++i) V[i] = (V0[i] + V1[i]) & m;
    or_ring_matmul(l, U, V, M, K, N, Z);                               /* Eq. 2 */
    for (int64_t i = 0; i < M * N; ++i) Z1[i] = (Z[i] - Z0[i]) & m;   /* Eq. 3 */
    free(U); free(V); free(Z);
}

EXPORT void or_hadamard_triplet_gen(int l, uint64_t seed, uint64_t call_id, int64_t n,
                                    uint64_t *U0, uint64_t *U1, uint64_t *V0, uint64_t *V1,
                                    uint64_t *Z0, uint64_t *Z1) {
    uint64_t m = ring_mask(l);
    dprg(l, seed, TAG('U', '0', 0, 0), call_id, 0, n, U0);
    dprg(l, seed, TAG('U', '1', 0, 0), call_id, 0, n, U1);
    dprg(l, seed, TAG('V', '0', 0, 0), call_id, 0, n, V0);
    dprg(l, seed, TAG('V', '1', 0, 0), call_id, 0, n, V1);
    dprg(l, seed, TAG('Z', '0', 0, 0), call_id, 0, n, Z0);
    for (int64_t i = 0; i < n; ++i) Z1[i] = (((U0[i] + U1[i]) * (V0[i] + V1[i])) - Z0[i]) & m;
}

/* ------------------------------------------------------------------------------------------ */
/* Beaver matmul, Eqs. 4-6, simulated for both parties.                       */
/*   Eq. 4: E_i = A_i - U_i, F_i = B_i - V_i        Eq. 5: E = E_0 + E_1, F = F_0 + F_1        */
/*   form 0 (canonical, R2 = BASELINE north_star): C_i = i.E.F + E.V_i + U_i.F + Z_i  */
/*   form 1 (paper Eq. 6):                                  C_i = (-i).E.F + A_i.F + E.B_i + Z_i */
/* Then optional SecureML local truncation by `trunc` bits (R7).  Trace outputs are nullable.  */
/* ------------------------------------------------------------------------------------------ */
EXPORT void or_truncate(int l, int party, uint64_t *x, int64_t n, int d);

EXPORT void or_beaver_matmul(int l, int form, const uint64_t *A0, const uint64_t *A1,
                             const uint64_t *B0, const uint64_t *B1, const uint64_t *U0,
                             const uint64_t *U1, const uint64_t *V0, const uint64_t *V1,
                             const uint64_t *Z0, const uint64_t *Z1, int64_t M, int64_t K,
                             int64_t N, int trunc, uint64_t *C0, uint64_t *C1,
                             uint64_t *tE0, uint64_t *tE1, uint64_t *tE, uint64_t *tF0,
                             uint64_t *tF1, uint64_t *tF) {
    uint64_t m = ring_mask(l);
    const uint64_t *A[2] = {A0, A1}, *B[2] = {B0, B1}, *U[2] = {U0, U1}, *V[2] = {V0, V1};
    const uint64_t *Z[2] = {Z0, Z1};
    uint64_t *C[2] = {C0, C1};
    uint64_t *Ei[2], *Fi[2];
    for (int i = 0; i < 2; ++i) { /* Eq. 4, party i */
        Ei[i] = malloc(sizeof(uint64_t) * M * K);
        Fi[i] = malloc(sizeof(uint64_t) * K * N);
        for (int64_t t = 0; t < M * K; ++t) Ei[i][t] = (A[i][t] - U[i][t]) & m;
        for (int64_t t = 0; t < K * N; ++t) Fi[i][t] = (B[i][t] - V[i][t]) & m;
    }
    uint64_t *E = malloc(sizeof(uint64_t) * M * K), *F = malloc(sizeof(uint64_t) * K * N);
    for (int64_t t = 0; t < M * K; ++t) E[t] = (Ei[0][t] + Ei[1][t]) & m; /* Eq. 5 (opening) */
    for (int64_t t = 0; t < K * N; ++t) F[t] = (Fi[0][t] + Fi[1][t]) & m;

    uint64_t *EF = malloc(sizeof(uint64_t) * M * N), *T1 = malloc(sizeof(uint64_t) * M * N);
    uint64_t *T2 = malloc(sizeof(uint64_t) * M * N);
    or_ring_matmul(l, E, F, M, K, N, EF);
    for (int i = 0; i < 2; ++i) {
        if (form == 0) {
            or_ring_matmul(l, E, V[i], M, K, N, T1);  /* E . V_i */
            or_ring_matmul(l, U[i], F, M, K, N, T2);  /* U_i . F */
            for (int64_t t = 0; t < M * N; ++t)
                C[i][t] = ((uint64_t)i * EF[t] + T1[t] + T2[t] + Z[i][t]) & m;
        } else {
            or_ring_matmul(l, A[i], F, M, K, N, T1);  /* A_i . F */
            or_ring_matmul(l, E, B[i], M, K, N, T2);  /* E . B_i */
            for (int64_t t = 0; t < M * N; ++t)
                C[i][t] = ((uint64_t)0 - (uint64_t)i * EF[t] + T1[t] + T2[t] + Z[i][t]) & m;
        }
        if (trunc > 0) or_truncate(l, i, C[i], M * N, trunc);
    }
    if (tE0) memcpy(tE0, Ei[0], sizeof(uint64_t) * M * K);
    if (tE1) memcpy(tE1, Ei[1], sizeof(uint64_t) * M * K);
    if (tE) memcpy(tE, E, sizeof(uint64_t) * M * K);
    if (tF0) memcpy(tF0, Fi[0], sizeof(uint64_t) * K * N);
    if (tF1) memcpy(tF1, Fi[1], sizeof(uint64_t) * K * N);
    if (tF) memcpy(tF, F, sizeof(uint64_t) * K * N);
    for (int i = 0; i < 2; ++i) { free(Ei[i]); free(Fi[i]); }
    free(E); free(F); free(EF); free(T1); free(T2);
}

/* Beaver Hadamard (elementwise) product, same algebra with . replaced by (.) elementwise.     */
EXPORT void or_beaver_hadamard(int l, const uint64_t *A0, const uint64_t *A1, const uint64_t *B0,
                               const uint64_t *B1, const uint64_t *U0, const uint64_t *U1,
                               const uint64_t *V0, const uint64_t *V1, const uint64_t *Z0,
                               const uint64_t *Z1, int64_t n, uint64_t *C0, uint64_t *C1) {
    uint64_t m = ring_mask(l);
    for (int64_t t = 0; t < n; ++t) {
        uint64_t e0 = A0[t] - U0[t], e1 = A1[t] - U1[t];
        uint64_t f0 = B0[t] - V0[t], f1 = B1[t] - V1[t];
        uint64_t e = (e0 + e1) & m, f = (f0 + f1) & m;
        C0[t] = (0 * e * f + e * V0[t] + U0[t] * f + Z0[t]) & m;
        C1[t] = (1 * e * f + e * V1[t] + U1[t] * f + Z1[t]) & m;
    }
}

/* ------------------------------------------------------------------------------------------ */
/* SecureML local share truncation (R7; not in PAPER.md): party 0: c >> d;                      */
/* party 1: -((-c) >> d); logical shifts on l-bit unsigned values.                            */
/* ------------------------------------------------------------------------------------------ */
EXPORT void or_truncate(int l, int party, uint64_t *x, int64_t n, int d) {
    uint64_t m = ring_mask(l);
    if (d <= 0) return;
    for (int64_t t = 0; t < n; ++t) {
        uint64_t v = x[t] & m;
        if (party == 0) x[t] = v >> d;
        else x[t] = ((uint64_t)0 - ((((uint64_t)0 - v) & m) >> d)) & m;
    }
}

/* ------------------------------------------------------------------------------------------ */
/* Secure MSB / DReLU (R9; PAPER.md only says Eq. 9 is computed "in GPUs", L178).              */
/* Dealer material per element e (all l-bit words):                                           */
/*   AND index t = 0..2L-1 (L = log2 l): a_i, b_i, c_0 from PRG tags {'a','0'+i,t}, ...,        */
/*   c_1 = ((a_0^a_1) & (b_0^b_1)) ^ c_0;                                                     */
/*   daBit: rB_i = PRG('R','0'+i) & 1; rA_0 = PRG('R','A'); rA_1 = (rB_0 ^ rB_1) - rA_0.        */
/* Material layout per party (uint64 words): [t][3][n] for (a,b,c) then rB[n], rA[n].           */
/* ------------------------------------------------------------------------------------------ */

/*
 * Secure MSB by a REDUCED Kogge-Stone carry prefix (R27, replacing the full-word R9
 * chain).  Only G[l-2] -- the carry into bit l-1 -- is needed, so after the first level only every
 * other prefix position matters, then every fourth, ...: level 1 gates the even bit positions
 * 2..l-2, after which the even positions are compacted into an l/2-bit word; every later level
 * gates the odd positions of the current word (G at every odd index, P at odd indices >= 3) and
 * compacts the odd positions.  For l = 64: 63 + 62 + 31 + 15 + 7 + 3 + 1 = 182 bit-ANDs instead of
 * 12 x 64, in the same 1 + log2(l) rounds.  Each AND is a boolean Beaver AND restricted to its gate
 * mask M: open e = (x ^ a) & M, f = (y ^ b) & M -- no bit outside M leaves a party.
 *
 * Material per element and party: 3 groups x (a, b, c) words + the daBit (r^B, r^A) = 11 words
 * (structure of arrays: word w of element e at mat[w * n + e]; group g at words 3g .. 3g + 2):
 *   group 0  round 0 (G = X0 & X1):  bits 0 .. l-2
 *   group 1  level 1: the G gates at their own (even) positions, the P gates shifted down by 1
 *            (odd positions): bits 1 .. l-2
 *   group 2  levels 2 .. log2(l): level j occupies a field of w_j = l / 2^(j-1) bits at offset
 *            sum of the previous widths; inside it the G gates at the odd positions and the P gates
 *            shifted down by 1 (even positions): field bits 1 .. w_j - 1
 * a_i = PRG('a', '0' + i, g) & mask_g, b_i likewise, c_0 = PRG('c', '0', g) & mask_g,
 * c_1 = ((a_0 ^ a_1) & (b_0 ^ b_1)) ^ c_0; r^B_i = PRG('R', '0' + i) & 1, r^A_0 = PRG('R', 'A'),
 * r^A_1 = (r^B_0 ^ r^B_1) - r^A_0.
 */
EXPORT int64_t or_msb_material_words(int l, int64_t n) { (void)l; return 11 * n; }

static uint64_t bits_mask(int lo, int hi) {   /* bits lo .. hi inclusive (hi < 64) */
    uint64_t m = 0;
    for (int b = lo; b <= hi; ++b) m |= (uint64_t)1 << b;
    return m;
}

static uint64_t msb_group_mask(int l, int g) {
    if (g == 0) return bits_mask(0, l - 2);
    if (g == 1) return bits_mask(1, l - 2);
    uint64_t m = 0;
    int off = 0;
    for (int w = l / 2; w >= 2; w /= 2) {
        m |= bits_mask(off + 1, off + w - 1);
        off += w;
    }
    return m;
}

EXPORT void or_msb_dealer(int l, uint64_t seed, uint64_t call_id, int64_t n, uint64_t *mat0,
                          uint64_t *mat1) {
    uint64_t m = ring_mask(l);
    uint64_t *mat[2] = {mat0, mat1};
    for (int g = 0; g < 3; ++g) {
        uint64_t gm = msb_group_mask(l, g);
        for (int i = 0; i < 2; ++i) {
            dprg(64, seed, TAG('a', '0' + i, g, 0), call_id, 0, n, mat[i] + ((int64_t)g * 3 + 0) * n);
            dprg(64, seed, TAG('b', '0' + i, g, 0), call_id, 0, n, mat[i] + ((int64_t)g * 3 + 1) * n);
        }
        uint64_t *c0 = mat0 + ((int64_t)g * 3 + 2) * n, *c1 = mat1 + ((int64_t)g * 3 + 2) * n;
        dprg(64, seed, TAG('c', '0', g, 0), call_id, 0, n, c0);
        for (int64_t e = 0; e < n; ++e) {
            for (int i = 0; i < 2; ++i) {
                mat[i][((int64_t)g * 3 + 0) * n + e] &= gm;
                mat[i][((int64_t)g * 3 + 1) * n + e] &= gm;
            }
            c0[e] &= gm;
            uint64_t a = mat0[((int64_t)g * 3 + 0) * n + e] ^ mat1[((int64_t)g * 3 + 0) * n + e];
            uint64_t b = mat0[((int64_t)g * 3 + 1) * n + e] ^ mat1[((int64_t)g * 3 + 1) * n + e];
            c1[e] = (a & b) ^ c0[e];
        }
    }
    int64_t off = 9 * n;
    dprg(l, seed, TAG('R', '0', 0, 0), call_id, 0, n, mat0 + off);
    dprg(l, seed, TAG('R', '1', 0, 0), call_id, 0, n, mat1 + off);
    for (int64_t e = 0; e < n; ++e) { mat0[off + e] &= 1; mat1[off + e] &= 1; }
    dprg(l, seed, TAG('R', 'A', 0, 0), call_id, 0, n, mat0 + off + n);
    for (int64_t e = 0; e < n; ++e)
        mat1[off + n + e] = ((mat0[off + e] ^ mat1[off + e]) - mat0[off + n + e]) & m;
}

/* One boolean Beaver AND for both parties of one element, restricted to the gate mask M:
 * open e = (x ^ a) & M, f = (y ^ b) & M; z_i = (i ? e&f : 0) ^ (e & b_i) ^ (a_i & f) ^ c_i. */
static void bool_and1(uint64_t M, uint64_t x0, uint64_t x1, uint64_t y0, uint64_t y1, uint64_t a0,
                      uint64_t a1, uint64_t b0, uint64_t b1, uint64_t c0, uint64_t c1, uint64_t *z0,
                      uint64_t *z1) {
    uint64_t e = ((x0 ^ a0) & M) ^ ((x1 ^ a1) & M);
    uint64_t f = ((y0 ^ b0) & M) ^ ((y1 ^ b1) & M);
    *z0 = (e & b0) ^ (a0 & f) ^ c0;
    *z1 = (e & f) ^ (e & b1) ^ (a1 & f) ^ c1;
}

/* Keep the bits at positions start, start + 2, start + 4, ... of a w-bit word, packed downwards. */
static uint64_t compact(uint64_t v, int w, int start) {
    uint64_t r = 0;
    int k = 0;
    for (int b = start; b < w; b += 2, ++k) r |= ((v >> b) & 1) << k;
    return r;
}

static uint64_t odd_bits(int lo, int w) {   /* odd positions >= lo below w */
    uint64_t m = 0;
    for (int b = 1; b < w; b += 2)
        if (b >= lo) m |= (uint64_t)1 << b;
    return m;
}

/*
 * MSB of x = x_0 + x_1 mod 2^l on boolean shares (P0 holds X0 := x_0 as (x_0, 0), P1 holds
 * X1 := x_1 as (0, x_1)), the reduced prefix of the header comment; msb = P_orig[l-1] ^ G[l-2].
 * Then B2A with the daBit: open c = msb ^ rB, [msb]^A_i = (i==0 ? c : 0) + (1 - 2c) rA_i.
 * Output: arithmetic shares of msb (0/1); optional boolean shares of msb (bit 0 of a word).
 */
EXPORT void or_secure_msb(int l, const uint64_t *x0, const uint64_t *x1, int64_t n,
                          const uint64_t *mat0, const uint64_t *mat1, uint64_t *msbA0,
                          uint64_t *msbA1, uint64_t *msbB0, uint64_t *msbB1) {
    uint64_t m = ring_mask(l);
    for (int64_t t = 0; t < n; ++t) {
#define W(i, g, k) ((i) == 0 ? mat0 : mat1)[((int64_t)(g) * 3 + (k)) * n + t]
        uint64_t X0 = x0[t] & m, X1 = x1[t] & m;
        uint64_t G[2], P[2];
        /* round 0: G = X0 & X1 on bits 0 .. l-2; P = X0 ^ X1 (local) */
        bool_and1(bits_mask(0, l - 2), X0, 0, 0, X1, W(0, 0, 0), W(1, 0, 0), W(0, 0, 1), W(1, 0, 1),
                  W(0, 0, 2), W(1, 0, 2), &G[0], &G[1]);
        P[0] = X0; P[1] = X1;
        /* level 1 (shift 1): gates at the even positions 2 .. l-2; the group-1 word carries the
         * G material there and the P material shifted down by one */
        {
            uint64_t MG = 0;
            for (int b = 2; b <= l - 2; b += 2) MG |= (uint64_t)1 << b;
            uint64_t zG[2], zP[2], aG[2], bG[2], cG[2], aP[2], bP[2], cP[2];
            for (int i = 0; i < 2; ++i) {
                aG[i] = W(i, 1, 0) & MG; aP[i] = (W(i, 1, 0) << 1) & MG;
                bG[i] = W(i, 1, 1) & MG; bP[i] = (W(i, 1, 1) << 1) & MG;
                cG[i] = W(i, 1, 2) & MG; cP[i] = (W(i, 1, 2) << 1) & MG;
            }
            bool_and1(MG, P[0], P[1], G[0] << 1, G[1] << 1, aG[0], aG[1], bG[0], bG[1], cG[0], cG[1], &zG[0], &zG[1]);
            bool_and1(MG, P[0], P[1], P[0] << 1, P[1] << 1, aP[0], aP[1], bP[0], bP[1], cP[0], cP[1], &zP[0], &zP[1]);
            for (int i = 0; i < 2; ++i) {
                G[i] = compact(G[i] ^ zG[i], l, 0);
                P[i] = compact(zP[i], l, 0);
            }
        }
        /* levels 2 .. log2(l) on the compacted words: gates at the odd positions (P at >= 3) */
        int off = 0;
        for (int w = l / 2; w >= 2; w /= 2) {
            uint64_t MG = odd_bits(1, w), MP = odd_bits(3, w), fm = (w == 64) ? ~(uint64_t)0 : (((uint64_t)1 << w) - 1);
            uint64_t zG[2], zP[2], aG[2], bG[2], cG[2], aP[2], bP[2], cP[2];
            for (int i = 0; i < 2; ++i) {
                uint64_t A = (W(i, 2, 0) >> off) & fm, Bw = (W(i, 2, 1) >> off) & fm, Cw = (W(i, 2, 2) >> off) & fm;
                aG[i] = A & MG; aP[i] = (A << 1) & MP;
                bG[i] = Bw & MG; bP[i] = (Bw << 1) & MP;
                cG[i] = Cw & MG; cP[i] = (Cw << 1) & MP;
            }
            bool_and1(MG, P[0], P[1], G[0] << 1, G[1] << 1, aG[0], aG[1], bG[0], bG[1], cG[0], cG[1], &zG[0], &zG[1]);
            bool_and1(MP, P[0], P[1], P[0] << 1, P[1] << 1, aP[0], aP[1], bP[0], bP[1], cP[0], cP[1], &zP[0], &zP[1]);
            for (int i = 0; i < 2; ++i) {
                G[i] = compact(G[i] ^ zG[i], w, 1);
                P[i] = compact(zP[i], w, 1);
            }
            off += w;
        }
#undef W
        uint64_t b0 = ((X0 >> (l - 1)) & 1) ^ (G[0] & 1); /* P_orig share 0 = x_0 */
        uint64_t b1 = ((X1 >> (l - 1)) & 1) ^ (G[1] & 1); /* P_orig share 1 = x_1 */
        if (msbB0) msbB0[t] = b0;
        if (msbB1) msbB1[t] = b1;
        int64_t doff = 9 * n;
        uint64_t c = (b0 ^ mat0[doff + t]) ^ (b1 ^ mat1[doff + t]); /* B2A opening */
        uint64_t s = (1 - 2 * c) & m;
        msbA0[t] = (c + s * mat0[doff + n + t]) & m;
        msbA1[t] = (s * mat1[doff + n + t]) & m;
    }
}

/* ------------------------------------------------------------------------------------------ */
/* CSR codec of PAPER.md L228 (compressed transmission of the inter-epoch delta, Eqs. 10-12).  */
/* Delta = cur - prev (mod 2^l), viewed as rows x cols.  CSR iff 4*nnz <= rows*cols (>= 75%   */
/* zeros), else dense.  Returns nnz; row_ptr[rows+1], col_idx[nnz], vals[nnz] filled for CSR. */
/* ------------------------------------------------------------------------------------------ */
EXPORT int64_t or_delta_csr_encode(int l, const uint64_t *cur, const uint64_t *prev, int64_t rows,
                                   int64_t cols, int32_t *is_csr, int32_t *row_ptr,
                                   int32_t *col_idx, uint64_t *vals, uint64_t *dense) {
    uint64_t m = ring_mask(l);
    int64_t nnz = 0;
    for (int64_t t = 0; t < rows * cols; ++t) nnz += ((cur[t] - prev[t]) & m) != 0;
    *is_csr = (4 * nnz <= rows * cols);
    if (*is_csr) {
        int64_t k = 0;
        row_ptr[0] = 0;
        for (int64_t r = 0; r < rows; ++r) {
            for (int64_t c = 0; c < cols; ++c) {
                uint64_t d = (cur[r * cols + c] - prev[r * cols + c]) & m;
                if (d) { col_idx[k] = (int32_t)c; vals[k] = d; ++k; }
            }
            row_ptr[r + 1] = (int32_t)k;
        }
    } else {
        for (int64_t t = 0; t < rows * cols; ++t) dense[t] = (cur[t] - prev[t]) & m;
    }
    return nnz;
}

EXPORT void or_delta_csr_apply(int l, int64_t rows, int64_t cols, int32_t is_csr,
                               const int32_t *row_ptr, const int32_t *col_idx, const uint64_t *vals,
                               const uint64_t *dense, uint64_t *target) {
    uint64_t m = ring_mask(l);
    if (is_csr) {
        for (int64_t r = 0; r < rows; ++r)
            for (int32_t k = row_ptr[r]; k < row_ptr[r + 1]; ++k)
                target[r * cols + col_idx[k]] = (target[r * cols + col_idx[k]] + vals[k]) & m;
    } else {
        for (int64_t t = 0; t < rows * cols; ++t) target[t] = (target[t] + dense[t]) & m;
    }
}

/* ------------------------------------------------------------------------------------------ */
/* One-round secure comparison by function secret sharing (R22).      */
/* Distributed comparison function (DCF) of Boyle, Chandran, Gilboa, Gupta, Ishai, Kumar and    */
/* Rathee, "Function Secret Sharing for Mixed-Mode and Fixed-Point Secure Computation"          */
/* (EUROCRYPT 2021), Fig. 1: f_{alpha,beta}(x) = beta if x < alpha else 0 over n-bit inputs      */
/* (bits taken most significant first), output group Z_{2^l}, seeds of lambda = 128 bits.       */
/* The paper only says Eq. 9 is computed "in GPUs"; this is the one-round       */
/* alternative to the Kogge-Stone A2B of R9.                                                    */
/* ------------------------------------------------------------------------------------------ */
typedef struct { uint64_t lo, hi; } seed128;

/* G: {0,1}^128 -> (s^L, v^L, t^L, s^R, v^R, t^R): one ChaCha20 block keyed by the seed (16 bytes
 * little endian || 16 zero bytes), counter 0, nonce = tag "DCFG" || 8 zero bytes.  Words 0-3 s^L,
 * 4-7 s^R, 8-9 v^L, 10-11 v^R (little endian u64, reduced mod 2^l), bit 0 of word 12 t^L, of 13 t^R. */
static void dcf_G(int l, seed128 s, seed128 *sL, uint64_t *vL, int *tL, seed128 *sR, uint64_t *vR, int *tR) {
    uint32_t key[8] = {(uint32_t)s.lo, (uint32_t)(s.lo >> 32), (uint32_t)s.hi, (uint32_t)(s.hi >> 32), 0, 0, 0, 0};
    uint32_t nonce[3] = {0x47464344u /* "DCFG" */, 0, 0};
    uint32_t w[16];
    or_chacha20_block(key, 0, nonce, w);
    uint64_t m = ring_mask(l);
    sL->lo = (uint64_t)w[0] | ((uint64_t)w[1] << 32);
    sL->hi = (uint64_t)w[2] | ((uint64_t)w[3] << 32);
    sR->lo = (uint64_t)w[4] | ((uint64_t)w[5] << 32);
    sR->hi = (uint64_t)w[6] | ((uint64_t)w[7] << 32);
    *vL = ((uint64_t)w[8] | ((uint64_t)w[9] << 32)) & m;
    *vR = ((uint64_t)w[10] | ((uint64_t)w[11] << 32)) & m;
    *tL = (int)(w[12] & 1);
    *tR = (int)(w[13] & 1);
}

static uint64_t convert(int l, seed128 s) { return s.lo & ring_mask(l); }   /* Convert_G: low word */
static inline uint64_t neg_if(int t, uint64_t v, uint64_t m) { return (t ? (0 - v) : v) & m; }

/* DCF key words (per party): [0] seed.lo, [1] seed.hi, then per level i = 1..n: s_CW.lo, s_CW.hi,
 * V_CW, t_CW^L | t_CW^R << 1; then CW^(n+1).  4n + 3 words. */
EXPORT int64_t or_dcf_key_words(int n_bits) { return 4 * (int64_t)n_bits + 3; }

/* Gen(1^lambda, alpha, beta) of Fig. 1 with the two root seeds given (drawn by the caller's PRG). */
EXPORT void or_dcf_gen(int l, int n_bits, uint64_t alpha, uint64_t beta, uint64_t s0lo, uint64_t s0hi,
                       uint64_t s1lo, uint64_t s1hi, uint64_t *k0, uint64_t *k1) {
    uint64_t m = ring_mask(l);
    seed128 s[2] = {{s0lo, s0hi}, {s1lo, s1hi}};
    int t[2] = {0, 1};
    uint64_t Va = 0;
    k0[0] = s0lo; k0[1] = s0hi; k1[0] = s1lo; k1[1] = s1hi;
    for (int i = 1; i <= n_bits; ++i) {
        seed128 sL[2], sR[2];
        uint64_t vL[2], vR[2];
        int tL[2], tR[2];
        for (int b = 0; b < 2; ++b) dcf_G(l, s[b], &sL[b], &vL[b], &tL[b], &sR[b], &vR[b], &tR[b]);
        int ai = (int)((alpha >> (n_bits - i)) & 1);               /* alpha_i, MSB first */
        /* Keep = the child on alpha's path, Lose = the other one */
        seed128 *sKeep = ai ? sR : sL, *sLose = ai ? sL : sR;
        uint64_t *vKeep = ai ? vR : vL, *vLose = ai ? vL : vR;
        int *tKeep = ai ? tR : tL;
        seed128 scw = {sLose[0].lo ^ sLose[1].lo, sLose[0].hi ^ sLose[1].hi};
        uint64_t Vcw = neg_if(t[1], (vLose[1] - vLose[0] - Va) & m, m);
        if (ai == 1) Vcw = (Vcw + neg_if(t[1], beta, m)) & m;      /* Lose = L: x < alpha below here */
        Va = (Va - vKeep[1] + vKeep[0] + neg_if(t[1], Vcw, m)) & m;
        int tcwL = tL[0] ^ tL[1] ^ ai ^ 1, tcwR = tR[0] ^ tR[1] ^ ai;
        int tcwKeep = ai ? tcwR : tcwL;
        int64_t o = 2 + 4 * (int64_t)(i - 1);
        k0[o] = k1[o] = scw.lo;
        k0[o + 1] = k1[o + 1] = scw.hi;
        k0[o + 2] = k1[o + 2] = Vcw;
        k0[o + 3] = k1[o + 3] = (uint64_t)(tcwL | (tcwR << 1));
        for (int b = 0; b < 2; ++b) {
            seed128 ns = sKeep[b];
            if (t[b]) { ns.lo ^= scw.lo; ns.hi ^= scw.hi; }
            int nt = tKeep[b] ^ (t[b] & tcwKeep);
            s[b] = ns;
            t[b] = nt;
        }
    }
    uint64_t last = neg_if(t[1], (convert(l, s[1]) - convert(l, s[0]) - Va) & m, m);
    k0[2 + 4 * (int64_t)n_bits] = k1[2 + 4 * (int64_t)n_bits] = last;
}

/* Eval(b, k_b, x) of Fig. 1: party b's additive share of f_{alpha,beta}(x). */
EXPORT uint64_t or_dcf_eval(int l, int n_bits, int b, const uint64_t *k, uint64_t x) {
    uint64_t m = ring_mask(l);
    seed128 s = {k[0], k[1]};
    int t = b;
    uint64_t V = 0;
    for (int i = 1; i <= n_bits; ++i) {
        int64_t o = 2 + 4 * (int64_t)(i - 1);
        seed128 scw = {k[o], k[o + 1]};
        uint64_t Vcw = k[o + 2];
        int tcwL = (int)(k[o + 3] & 1), tcwR = (int)((k[o + 3] >> 1) & 1);
        seed128 sL, sR;
        uint64_t vL, vR;
        int tL, tR;
        dcf_G(l, s, &sL, &vL, &tL, &sR, &vR, &tR);
        if (t) {
            sL.lo ^= scw.lo; sL.hi ^= scw.hi; tL ^= tcwL;
            sR.lo ^= scw.lo; sR.hi ^= scw.hi; tR ^= tcwR;
        }
        int xi = (int)((x >> (n_bits - i)) & 1);
        if (!xi) {
            V = (V + neg_if(b, (vL + (t ? Vcw : 0)) & m, m)) & m;
            s = sL; t = tL;
        } else {
            V = (V + neg_if(b, (vR + (t ? Vcw : 0)) & m, m)) & m;
            s = sR; t = tR;
        }
    }
    uint64_t last = k[2 + 4 * (int64_t)n_bits];
    V = (V + neg_if(b, (convert(l, s) + (t ? last : 0)) & m, m)) & m;
    return V;
}

/*
 * FSS DReLU material (R22), per element e and party b, as fss_words(l) = 4(l-1) + 5
 * words in structure-of-arrays order (word w of element e at mat_b[w * n + e]):
 *   w = 0: r_b        additive share of the input mask r = PRG(seed, "FR", id)[e]
 *                     (r_0 = PRG("F0"), r_1 = r - r_0)
 *   w = 1: sA_b       additive share of s = MSB(r)  (sA_0 = PRG("FS"), sA_1 = s - sA_0)
 *   w = 2..:          DCF key of f_{alpha,beta} with n = l - 1 input bits, alpha = r mod 2^(l-1),
 *                     beta = 1 - 2s (mod 2^l); root seeds (PRG("K0")[2e], [2e+1]) and
 *                     (PRG("K1")[2e], [2e+1]).
 */
EXPORT int64_t or_fss_words(int l) { return 4 * (int64_t)(l - 1) + 5; }

EXPORT void or_fss_dealer(int l, uint64_t seed, uint64_t call_id, int64_t n, uint64_t *mat0, uint64_t *mat1) {
    uint64_t m = ring_mask(l);
    int nb = l - 1;
    int64_t kw = or_dcf_key_words(nb);
    uint64_t *r = malloc(sizeof(uint64_t) * n), *r0 = malloc(sizeof(uint64_t) * n), *sa0 = malloc(sizeof(uint64_t) * n);
    uint64_t *K0 = malloc(sizeof(uint64_t) * 2 * n), *K1 = malloc(sizeof(uint64_t) * 2 * n);
    dprg(l, seed, 0x00005246u /* "FR" */, call_id, 0, n, r);
    dprg(l, seed, 0x00003046u /* "F0" */, call_id, 0, n, r0);
    dprg(l, seed, 0x00005346u /* "FS" */, call_id, 0, n, sa0);
    dprg(64, seed, 0x0000304Bu /* "K0" */, call_id, 0, 2 * n, K0);
    dprg(64, seed, 0x0000314Bu /* "K1" */, call_id, 0, 2 * n, K1);
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < n; ++e) {
        uint64_t k0[4 * 64 + 3], k1[4 * 64 + 3];
        uint64_t sbit = (r[e] >> (l - 1)) & 1;
        uint64_t alpha = r[e] & (((uint64_t)1 << nb) - 1);
        uint64_t beta = (1 - 2 * sbit) & m;
        or_dcf_gen(l, nb, alpha, beta, K0[2 * e], K0[2 * e + 1], K1[2 * e], K1[2 * e + 1], k0, k1);
        mat0[e] = r0[e];
        mat1[e] = (r[e] - r0[e]) & m;
        mat0[n + e] = sa0[e];
        mat1[n + e] = (sbit - sa0[e]) & m;
        for (int64_t w = 0; w < kw; ++w) {
            mat0[(2 + w) * n + e] = k0[w];
            mat1[(2 + w) * n + e] = k1[w];
        }
    }
    free(r); free(r0); free(sa0); free(K0); free(K1);
}

/*
 * FSS DReLU, both parties (R22).  Round 1 (the only opening): xhat = (x_0 + r_0) +
 * (x_1 + r_1) = x + r.  Then locally, with c = MSB(xhat) and xhat' = xhat mod 2^(l-1):
 *   MSB(x) = c XOR s XOR [xhat' < r']   (x = xhat - r: a borrow out of the low l-1 bits flips the MSB)
 *   [s XOR borrow]_b = sA_b + Eval(b, k_b, xhat')            (the DCF pays beta = 1 - 2s)
 *   [MSB]_b = c ? [b = 0] - [s XOR borrow]_b : [s XOR borrow]_b ;  DReLU_b = [b = 0] - [MSB]_b.
 * Outputs arithmetic shares of DReLU(x) = 1{x >= 0} (signed), and the opened xhat (trace).
 */
EXPORT void or_fss_drelu(int l, const uint64_t *x0, const uint64_t *x1, int64_t n, const uint64_t *mat0,
                         const uint64_t *mat1, uint64_t *d0, uint64_t *d1, uint64_t *xhat_out) {
    uint64_t m = ring_mask(l);
    int nb = l - 1;
    int64_t kw = or_dcf_key_words(nb);
    const uint64_t *mat[2] = {mat0, mat1};
    uint64_t *d[2] = {d0, d1};
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < n; ++e) {
        uint64_t xhat = ((x0[e] + mat0[e]) + (x1[e] + mat1[e])) & m;   /* Eq. 4-5 style opening */
        if (xhat_out) xhat_out[e] = xhat;
        uint64_t c = (xhat >> (l - 1)) & 1;
        uint64_t xlow = xhat & (((uint64_t)1 << nb) - 1);
        uint64_t k[4 * 64 + 3];
        for (int b = 0; b < 2; ++b) {
            for (int64_t w = 0; w < kw; ++w) k[w] = mat[b][(2 + w) * n + e];
            uint64_t sb = (mat[b][n + e] + or_dcf_eval(l, nb, b, k, xlow)) & m;
            uint64_t msb = c ? (((uint64_t)(b == 0)) - sb) & m : sb;
            d[b][e] = (((uint64_t)(b == 0)) - msb) & m;
        }
    }
}

EXPORT int or_num_threads(void) {
#ifdef _OPENMP
    extern int omp_get_max_threads(void);
    return omp_get_max_threads();
#else
    return 1;
#endif
}
