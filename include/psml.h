/*
 * psml.h -- C ABI of the B200-native ParSecureML hot path (libpsml.so).
 *
 * What the library computes: the two-party Beaver-triplet secure matrix multiplication of
 * PAPER.md Sec. 2.2 (L65-L78, Eqs. 1-6) on additive secret shares in the ring Z_{2^l}
 * (l = 64 or 32, SecureML fixed point with `frac_bits` = 13), in the one-GEMM shape of
 * Sec. 4.2 (L164-L176, Eqs. 7-8), followed by SecureML local share truncation, the secure
 * activations (Eq. 9, and ReLU) and the gradient/update steps of secure linear and
 * logistic regression, MLP and CNN training and inference (Sec. 4.3; Sec. 7.1,
 * L284-L295).  Readings where the paper is silent are DESIGN.md R1..R18.
 *
 * Conventions (every entry point):
 *  - All tensor arguments are CALLER-OWNED DEVICE pointers (CUDA global memory of the current
 *    device) unless the parameter name ends in `_host`.  Row-major, contiguous.  Element type
 *    uint64_t for l = 64 and uint32_t for l = 32 (a residue mod 2^l); `double` for plaintext.
 *    Base addresses must be 16-byte aligned (PSML_ERR_ALIGN otherwise).
 *  - "Pair" arguments `x[2]` hold party 0's and party 1's share of the same tensor.  This is the
 *    co-resident pair engine: both servers of PAPER.md Fig. 1b run on one GPU and an "opening"
 *    (Eq. 5) reads the peer's masked message from its send buffer in HBM.  Every protocol round
 *    is one kernel that opens the previous round's messages and emits the next round's, so the
 *    message boundary is explicit.
 *  - Every call enqueues work on `stream` and returns immediately.  Argument errors are
 *    reported synchronously (PSML_ERR_INVALID / _SHAPE / _ALIGN / _UNSUPPORTED) with nothing
 *    enqueued; CUDA launch failures return PSML_ERR_CUDA.  psml_last_error() gives a
 *    thread-local human-readable message for the last failing call.  No C++ exception crosses
 *    the ABI.  Contexts and models are not thread-safe: one host thread per context.
 *  - Randomness: the dealer and the client draw from ChaCha20 in counter mode (RFC 8439
 *    block function; R1) keyed by (seed, 4-byte role tag, 64-bit call id), so every
 *    share and triplet is reproducible bit-for-bit by the CPU oracle.
 */
#ifndef PSML_H_
#define PSML_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define PSML_ABI_VERSION 1

typedef struct CUstream_st *psml_stream; /* a cudaStream_t; NULL = legacy default stream */

typedef enum {
    PSML_OK = 0,
    PSML_ERR_INVALID = 1,     /* bad enum / null pointer / l not in {32, 64} / party not 0,1 */
    PSML_ERR_SHAPE = 2,       /* non-positive or inconsistent dimensions, bits >= l          */
    PSML_ERR_ALIGN = 3,       /* pointer not 16-byte aligned                                  */
    PSML_ERR_UNSUPPORTED = 4, /* configuration not built (e.g. no sm_100 device)              */
    PSML_ERR_CUDA = 5,        /* a CUDA runtime/driver call or kernel launch failed           */
    PSML_ERR_NOMEM = 6,       /* device allocation failed                                     */
    PSML_ERR_STATE = 7,       /* object used in the wrong state (e.g. step without deal)      */
    PSML_ERR_NCCL = 8         /* a transport exchange (NCCL call or host callback) failed     */
} psml_status;

/* The ring Z_{2^l} and the fixed-point scale (SecureML: frac_bits = 13).  DESIGN.md R3. */
typedef struct {
    int32_t l;         /* 32 or 64 */
    int32_t frac_bits; /* 0 <= frac_bits < l */
} psml_ring;

typedef struct psml_ctx_s *psml_ctx;     /* one per (GPU, host thread); owns workspaces */
typedef struct psml_model_s *psml_model; /* weight shares + dealer pool of one model      */

/* ------------------------------------------------------------------------------------------ */
/* Library / device                                                                            */
/* ------------------------------------------------------------------------------------------ */
int32_t psml_abi_version(void);
const char *psml_last_error(void);
/* Writes the current device's SM count and compute capability.  Fails with
 * PSML_ERR_UNSUPPORTED if no CUDA device is visible. */
psml_status psml_device_info(int32_t *sm_count, int32_t *cc_major, int32_t *cc_minor);
/* Number of kernels this process has launched through the library (for bench accounting). */
uint64_t psml_kernel_launch_count(void);

/* Kernel-class timing for bench.py's roofline (off by default).  While enabled for class `cls`,
 * every library launch of that class is bracketed by CUDA events on its own stream, and its
 * algorithmic work is accumulated: ring GEMMs count ring multiply-adds (M*N*K' per party),
 * the elementwise classes count algorithmic HBM bytes (each word read + written once).
 * cls: 0 CUDA-core ring GEMM, 1 tcgen05 limb GEMM, 2 MSB/ReLU/Eq. 9 round kernels,
 *      3 Hadamard rounds, 4 dealer PRG kernels, 5 Beaver masking, -1 = disable.
 * psml_prof_read synchronizes the device, returns the totals and resets them. */
psml_status psml_prof_enable(int32_t cls);
psml_status psml_prof_read(double *total_ms, int64_t *launches, double *work);
/* Measurement utility (synchronous, not part of the hot path): the device's ring multiply-add
 * throughput in Z_2^l on CUDA cores, measured with a register-only kernel of independent
 * acc = acc + a * b chains (l = 64: IMAD.WIDE.U32 + 2 IMAD per MAC, the ring GEMM inner loop;
 * l = 32: one IMAD) on every SM -- the ALU roofline denominator of the CUDA-core ring GEMMs. */
psml_status psml_bench_mac_peak(int32_t l, double *ring_macs_per_s);

/* ------------------------------------------------------------------------------------------ */
/* Context                                                                                     */
/* ------------------------------------------------------------------------------------------ */
/* gemm_backend: 0 = auto (tcgen05 limb GEMM where the shape pays, CUDA-core otherwise),
 *               1 = CUDA-core only, 2 = tcgen05 only (PSML_ERR_UNSUPPORTED if not sm_100). */
psml_status psml_ctx_create(psml_ring ring, int32_t gemm_backend, psml_ctx *out);
psml_status psml_ctx_destroy(psml_ctx ctx);

/* Execution options of a context (explicit arguments, no process globals).  Every field
 * selects between bit-identical implementations (tested against each other and the oracle); the
 * defaults are the measured fastest.  A call on a context -- or on a model created
 * from it -- runs with that context's options.  psml_options_default fills the defaults. */
typedef struct {
    int32_t seg_backend;   /* training-step Beaver products: 0 auto (tcgen05 for groups of >= 2^25
                              ring MACs on sm_100), 1 CUDA cores only, 2 tcgen05 wherever eligible */
    int32_t pdl;           /* programmatic dependent launch between step kernels (1)          */
    int32_t fused_open;    /* eager Beaver matmul: 0 mask round then GEMM (default), 1 mask fused
                              into the GEMM's operand loads                                    */
    int32_t fused_step;    /* co-resident MLP-family step: 1 producers open their consumers'
                              operands (default), 0 one open pass per product                 */
    int32_t fused_dealer;  /* 1 the step's dealer as two launches (default), 0 per item        */
    int32_t deal_split;    /* pipelined graph: dealer PRG on two branches (1) or one (0)       */
    int32_t deal_after;    /* pipelined graph: fork the dealer after this many online stages (1) */
    int32_t gradw_branch;  /* weight gradients on their own graph branch (1)                  */
    int32_t simt_cluster;  /* CUDA-core products: 1 cluster split-K kernel, 0 16 x 16 small tile */
    int32_t rows_kernel;   /* CNN tall-skinny conv products: 1 rows kernel, 0 small tile        */
    int32_t msb_chain;     /* MSB chain: 0 one lane-pair launch, 1 one kernel per round        */
    int32_t conv_gw;       /* CNN weight gradient: 1 per-image kernel, 0 generic im2col GEMM    */
    int32_t split_fused;   /* split deployment over a peer transport: 1 each activation is ONE
                              kernel with its 9 rounds' exchanges fused over peer memory, 0 one
                              kernel + one exchange per round                                   */
    int32_t deal_on_launch; /* pipelined graph: 1 = the dealer branch forks as soon as every CTA of
                              the first tcgen05 product is resident (a launch-completion edge),
                              so the product's SMs are taken before the dealer's grids; 0 = after
                              the deal_after-th online stage completes                          */
    int32_t tc_small;      /* stand-alone psml_ring_gemm / co-resident psml_secure_matmul in Z_2^64
                              (BASELINE config 5 at small n) on tcgen05: 1 auto = products whose
                              128 x 64 output tiles (x 2 parties) fit one wave of the SMs (two
                              waves at l = 64) and K' <= 16384 run on the in-kernel limb-split kernel (one launch,
                              cluster split-K over the whole GPU), larger ones on the limb-plane
                              kernels; 0 always the limb-plane kernels; 2 the in-kernel split
                              kernel wherever K' <= 16384                                       */
} psml_options;
psml_status psml_options_default(psml_options *out);
psml_status psml_ctx_set_options(psml_ctx ctx, const psml_options *opts);

/* ------------------------------------------------------------------------------------------ */
/* PRG / client side (the client partitions inputs into shares)       */
/* ------------------------------------------------------------------------------------------ */
/* out[i] = element (offset + i) of the ChaCha20 stream (seed, tag, call_id) reduced mod 2^l.
 * Element layout: l = 64 -> words (2j, 2j+1) of block e/8, j = e%8; l = 32 -> word e%16 of
 * block e/16 (R1).  `tag` packs a 4-byte role tag little-endian. */
psml_status psml_prg_fill(psml_ring ring, uint64_t seed, uint32_t tag, uint64_t call_id,
                          uint64_t offset, int64_t n, void *out, psml_stream stream);
/* v = round_half_even(x * 2^frac_bits) mod 2^l; x: n doubles (device).  DESIGN.md R3. */
psml_status psml_encode(psml_ring ring, const double *x, int64_t n, void *v, psml_stream stream);
/* x = signed(v) / 2^frac_bits. */
psml_status psml_decode(psml_ring ring, const void *v, int64_t n, double *x, psml_stream stream);
/* Additive sharing: x0 = PRG(seed, "SH", stream_id)[0..n), x1 = x - x0 (mod 2^l).
 * x may alias neither x0 nor x1. */
psml_status psml_share(psml_ring ring, uint64_t seed, uint64_t stream_id, const void *x,
                       int64_t n, void *x0, void *x1, psml_stream stream);
/* psml_encode then psml_share in one pass: x0 = PRG(seed, "SH", stream_id), x1 = encode(x) - x0.
 * x: n doubles (device).  Bit-identical to the two calls. */
psml_status psml_encode_share(psml_ring ring, uint64_t seed, uint64_t stream_id, const double *x,
                              int64_t n, void *x0, void *x1, psml_stream stream);
/* Client encode + share straight from 8-bit pixels (image pixels 0..255):
 * x = q / den in fp64 (IEEE division), then exactly psml_encode_share.  q: n bytes (device).
 * Bit-identical to psml_encode_share on the float64 q / den.  den > 0 (255 for 8-bit images). */
psml_status psml_encode_share_u8(psml_ring ring, uint64_t seed, uint64_t stream_id, const uint8_t *q,
                                 int64_t n, double den, void *x0, void *x1, psml_stream stream);
/* Client encode + share of one-hot labels from class indices: Y[r][c] = (cls[r] == c), encoded
 * (1 -> 2^frac_bits, 0 -> 0) and shared like psml_encode_share on the float64 one-hot matrix
 * (rows x classes, row-major).  cls: rows bytes (device); a class index >= classes gives an
 * all-zero row. */
psml_status psml_encode_share_onehot(psml_ring ring, uint64_t seed, uint64_t stream_id,
                                     const uint8_t *cls, int64_t rows, int64_t classes, void *x0,
                                     void *x1, psml_stream stream);
/* x = x0 + x1 mod 2^l (client-side reconstruction). */
psml_status psml_reconstruct(psml_ring ring, const void *x0, const void *x1, int64_t n, void *x,
                             psml_stream stream);

/* ------------------------------------------------------------------------------------------ */
/* Dealer (offline phase; Eqs. 2-3, Fig. 4; R4)                        */
/* ------------------------------------------------------------------------------------------ */
/* Matrix triplet for an M x K by K x N product: U_i (MxK), V_i (KxN), Z_i (MxN).
 * U_0 = PRG("U0"), U_1 = PRG("U1"), V_0 = PRG("V0"), V_1 = PRG("V1"), Z_0 = PRG("Z0"),
 * Z_1 = (U_0 + U_1)(V_0 + V_1) - Z_0, all streams keyed by (seed, call_id).  Uses the ctx's
 * ring GEMM for Z. */
psml_status psml_triplet_gen(psml_ctx ctx, uint64_t seed, uint64_t call_id, int64_t M, int64_t K,
                             int64_t N, void *const U[2], void *const V[2], void *const Z[2],
                             psml_stream stream);
/* Rows [row0, row0 + M) of the M_total x K by K x N triplet psml_triplet_gen(seed, call_id,
 * M_total, K, N) would deal: U_i rows (elements row0*K .. of the "U0"/"U1" streams), the WHOLE V_i
 * and Z_i rows (Z_0 elements row0*N .., Z_1 = U[rows] V - Z_0[rows]); bit-identical to slicing the
 * full triplet.  The M-row sharding of a secure product over data-parallel pairs (SURVEY 8(e)
 * config 5, R28): pair k deals its own rows, every pair opens the same F = B - V.
 * U_i: M x K, V_i: K x N, Z_i: M x N (device, caller-owned).  PSML_ERR_SHAPE unless
 * 0 <= row0, M > 0 and row0 + M <= M_total. */
psml_status psml_triplet_gen_rows(psml_ctx ctx, uint64_t seed, uint64_t call_id, int64_t M_total, int64_t row0,
                                  int64_t M, int64_t K, int64_t N, void *const U[2], void *const V[2],
                                  void *const Z[2], psml_stream stream);
/* Elementwise (Hadamard) triplet of n elements: same streams, Z_1 = (U_0+U_1)(V_0+V_1) - Z_0. */
psml_status psml_hadamard_triplet_gen(psml_ring ring, uint64_t seed, uint64_t call_id, int64_t n,
                                      void *const U[2], void *const V[2], void *const Z[2],
                                      psml_stream stream);
/* Words (of l bits) of MSB material per party for n elements: 11 n (R27). */
int64_t psml_msb_material_words(psml_ring ring, int64_t n);
/* Boolean AND triplets of the REDUCED Kogge-Stone prefix and the daBit for B2A (R27).
 * mat[i] layout (words, structure of arrays): for AND group g = 0, 1, 2: a_i[n], b_i[n], c_i[n]
 * (group 0: round 0 on bits 0..l-2; group 1: level 1, G material at the even positions 2..l-2 and
 * P material shifted down by one; group 2: levels 2..log2(l), level j in a field of l/2^(j-1) bits
 * at offset l - 2 l/2^(j-1), G material at its odd positions, P shifted down by one); then
 * rB_i[n] (bit), rA_i[n].  a_i = PRG('a','0'+i,g) & mask_g, b_i = PRG('b','0'+i,g) & mask_g,
 * c_0 = PRG('c','0',g) & mask_g, c_1 = ((a_0^a_1) & (b_0^b_1)) ^ c_0; rB_i = PRG('R','0'+i) & 1;
 * rA_0 = PRG('R','A'), rA_1 = (rB_0 ^ rB_1) - rA_0.  Streams keyed per R23. */
psml_status psml_msb_dealer(psml_ring ring, uint64_t seed, uint64_t call_id, int64_t n,
                            void *const mat[2], psml_stream stream);

/* ------------------------------------------------------------------------------------------ */
/* Server side: secure operations on share pairs                                               */
/* ------------------------------------------------------------------------------------------ */
#define PSML_TRANS_A 1    /* use A^T: A is stored K x M                                     */
#define PSML_TRANS_B 2    /* use B^T: B is stored N x K                                     */
#define PSML_PAPER_FORM 4 /* C_i = (-i)EF + A_i F + E B_i + Z_i (Eq. 6) instead of BJ form  */

/* Optional trace of the opened values (all device, nullable): E_i = op(A)_i - U_i (M x K),
 * F_i = op(B)_i - V_i (K x N) and the opened E = E_0 + E_1, F = F_0 + F_1 (Eqs. 4-5). */
typedef struct {
    void *E[2];
    void *E_open;
    void *F[2];
    void *F_open;
} psml_trace;

/* Beaver matmul (Eqs. 4-6 in the Eq. 8 shape): C_i = i.E.F + E.V_i + U_i.F + Z_i
 * (BJ canonical form) computed per party as ONE ring GEMM over the K-concatenation
 * [i.E + U_i | E] . [F ; V_i] + Z_i, then SecureML truncation by trunc_bits (0 = none).
 * A: M x K (or K x M with PSML_TRANS_A), B: K x N (or N x K), U_i: M x K, V_i: K x N,
 * Z_i, C_i: M x N.  C must not alias any input. */
psml_status psml_secure_matmul(psml_ctx ctx, const void *const A[2], const void *const B[2],
                               const void *const U[2], const void *const V[2],
                               const void *const Z[2], int64_t M, int64_t K, int64_t N,
                               int32_t flags, int32_t trunc_bits, void *const C[2],
                               const psml_trace *trace, psml_stream stream);
/* Split deployment: ONE party per process / GPU (Fig. 1b: two servers).  The Beaver
 * product becomes two calls around the caller's exchange of the masked messages:
 *  round 1  psml_beaver_mask: E_send = op(A)_i - U_i (M x K), F_send = op(B)_i - V_i (K x N)
 *           (Eq. 4); the caller sends E_send, F_send to the peer and receives the peer's
 *           E_recv, F_recv (e.g. NCCL send/recv over NVLink; uint64/uint32 words).
 *  round 2  psml_beaver_open_matmul: E = E_send + E_recv, F = F_send + F_recv (Eq. 5) opened
 *           inside the GEMM's operand loads, C_i = i.E.F + E.V_i + U_i.F + Z_i (Eq. 8 shape),
 *           then truncation by trunc_bits.  Bit-identical to psml_secure_matmul's party-i share.
 * Buffers are caller-owned device memory; the two calls must use the same shapes and flags. */
psml_status psml_beaver_mask(psml_ctx ctx, int32_t party, const void *A_i, const void *B_i,
                             const void *U_i, const void *V_i, int64_t M, int64_t K, int64_t N,
                             int32_t flags, void *E_send, void *F_send, psml_stream stream);
psml_status psml_beaver_open_matmul(psml_ctx ctx, int32_t party, const void *E_send,
                                    const void *E_recv, const void *F_send, const void *F_recv,
                                    const void *U_i, const void *V_i, const void *Z_i, int64_t M,
                                    int64_t K, int64_t N, int32_t trunc_bits, void *C_i,
                                    psml_stream stream);
/* Beaver Hadamard product of n elements: C_i = i.E.F + E.V_i + U_i.F + Z_i elementwise. */
psml_status psml_secure_hadamard(psml_ctx ctx, const void *const A[2], const void *const B[2],
                                 const void *const U[2], const void *const V[2],
                                 const void *const Z[2], int64_t n, int32_t trunc_bits,
                                 void *const C[2], psml_stream stream);
/* SecureML local truncation of one party's share in place: party 0: x >> bits;
 * party 1: -((-x) >> bits) (logical shifts on l-bit values; R7). */
psml_status psml_truncate(psml_ring ring, int32_t party, void *x_i, int64_t n, int32_t bits,
                          psml_stream stream);
/* Arithmetic shares of MSB(x) (0/1) by the reduced Kogge-Stone A2B (R27: only the gate bits that
 * reach the carry into bit l-1; 182 bit-ANDs at l = 64) + daBit B2A: 1 + log2(l) rounds of boolean
 * ANDs then 1 B2A round.  mat from psml_msb_dealer.  msbB (nullable): boolean shares. */
psml_status psml_secure_msb(psml_ctx ctx, const void *const x[2], int64_t n,
                            const void *const mat[2], void *const msbA[2], void *const msbB[2],
                            psml_stream stream);
/* ReLU(x) = x . (1 - MSB(x)) via one extra Beaver Hadamard (triplet U, V, Z of n elements).
 * drelu (nullable) receives the shares of 1 - MSB(x) (kept for backprop). */
psml_status psml_secure_relu(psml_ctx ctx, const void *const x[2], int64_t n,
                             const void *const mat[2], const void *const U[2],
                             const void *const V[2], const void *const Z[2], void *const y[2],
                             void *const drelu[2], psml_stream stream);
/* PAPER.md Eq. 9: f(x) = ReLU(x + 1/2) - ReLU(x - 1/2) = clamp(x + 1/2, 0, 1) on the grid.
 * mat: MSB material for 2n elements; U, V, Z: Hadamard triplet of 2n elements. */
psml_status psml_secure_eq9(psml_ctx ctx, const void *const x[2], int64_t n,
                            const void *const mat[2], const void *const U[2],
                            const void *const V[2], const void *const Z[2], void *const y[2],
                            psml_stream stream);

/* One-round secure comparison by function secret sharing (R22): the
 * distributed comparison function of Boyle et al. (EUROCRYPT 2021, Fig. 1) replaces the
 * 1 + log2(l)-round Kogge-Stone A2B of psml_secure_msb for DReLU.  Z_2^64 only
 * (PSML_ERR_UNSUPPORTED otherwise).  psml_fss_dealer writes, per element and party, 257 words in
 * structure-of-arrays order (word w of element e at mat[i][w * n + e]): the input-mask share r_i,
 * the share of s = MSB(r), the party's 128-bit DCF root seed and the 63 levels of correction words
 * + the final one (layout in fss.cuh; streams keyed by (seed, "FR"/"F0"/"FS"/"K0"/"K1", call_id)).
 * psml_fss_material_words(ring, n) = 257 n for l = 64, -1 otherwise.
 * psml_secure_drelu_fss: ONE opening (xhat = x + r), then each party evaluates its DCF key on the
 * low 63 bits of xhat: arithmetic shares of DReLU(x) = [x >= 0 signed] in drelu[2];
 * xhat_trace (nullable, device, n words) receives the opened value.  psml_secure_relu_fss adds
 * the Beaver Hadamard y = x . DReLU(x) (triplet U, V, Z of n elements), drelu nullable.
 * Split deployment: psml_fss_mask writes party i's message x_i + r_i; after the exchange
 * psml_fss_open_drelu opens xhat = msg_send + msg_recv and writes party i's DReLU share. */
int64_t psml_fss_material_words(psml_ring ring, int64_t n);
psml_status psml_fss_dealer(psml_ring ring, uint64_t seed, uint64_t call_id, int64_t n, void *const mat[2],
                            psml_stream stream);
psml_status psml_secure_drelu_fss(psml_ctx ctx, const void *const x[2], int64_t n, const void *const mat[2],
                                  void *const drelu[2], void *xhat_trace, psml_stream stream);
psml_status psml_secure_relu_fss(psml_ctx ctx, const void *const x[2], int64_t n, const void *const mat[2],
                                 const void *const U[2], const void *const V[2], const void *const Z[2],
                                 void *const y[2], void *const drelu[2], psml_stream stream);
psml_status psml_fss_mask(psml_ctx ctx, int32_t party, const void *x_i, int64_t n, const void *mat_i, void *msg,
                          psml_stream stream);
psml_status psml_fss_open_drelu(psml_ctx ctx, int32_t party, const void *msg_send, const void *msg_recv, int64_t n,
                                const void *mat_i, void *drelu_i, psml_stream stream);

/* Plain ring GEMM C = A . B mod 2^l (A: M x K, B: K x N, row-major) -- the config-5 sweep
 * kernel and the dealer's Z = U V.  Uses the ctx's backend choice. */
psml_status psml_ring_gemm(psml_ctx ctx, const void *A, const void *B, int64_t M, int64_t K,
                           int64_t N, void *C, psml_stream stream);

/* ------------------------------------------------------------------------------------------ */
/* Compressed transmission (Eqs. 10-12): delta of a party's masked message     */
/* against the previous opening, as CSR iff >= 75% zeros (4 nnz <= rows*cols), else dense.    */
/* ------------------------------------------------------------------------------------------ */
/* Writes *nnz_host and *is_csr_host (synchronizes `stream`).  CSR: row_ptr[rows+1] (int32),
 * col_idx[nnz] (int32), vals[nnz]; dense: dense[rows*cols].  All outputs are device buffers
 * of worst-case size sized by the caller. */
psml_status psml_delta_encode(psml_ctx ctx, const void *cur, const void *prev, int64_t rows,
                              int64_t cols, int32_t *row_ptr, int32_t *col_idx, void *vals,
                              void *dense, int64_t *nnz_host, int32_t *is_csr_host,
                              psml_stream stream);
/* target += delta (CSR or dense) mod 2^l. */
psml_status psml_delta_apply(psml_ctx ctx, int64_t rows, int64_t cols, int32_t is_csr,
                             const int32_t *row_ptr, const int32_t *col_idx, const void *vals,
                             const void *dense, void *target, psml_stream stream);

/* ------------------------------------------------------------------------------------------ */
/* Models: secure training / inference (Sec. 4.3, Sec. 7.1)      */
/* ------------------------------------------------------------------------------------------ */
/* PSML_SVM: linear SVM, hinge-loss minibatch subgradient with weight decay (PAPER.md L295 names
 * SVM trained by SMO; R24 reads it as the primal subgradient form that runs on the
 * Beaver / comparison primitives): z = X w; ind = [y z < 1]; gradW = X^T (-(y (.) ind)); labels
 * +-1.  Co-resident engine only. */
/* PSML_RNN: Elman RNN over rnn_steps = T steps (R25): dims = {D, H, C},
 * X: batch x (T D) (step t = columns t D .. (t+1) D), h_t = ReLU([x_t | h_{t-1}] . W_1) with W_1 of
 * (D + H) x H, yhat = Eq9(h_T . W_o) with W_o of H x C; trained by backpropagation through time
 * (the weight gradient of W_1 is the ring sum over t).  Co-resident engine only. */
typedef enum { PSML_LINREG = 0, PSML_LOGREG = 1, PSML_MLP = 2, PSML_CNN = 3, PSML_SVM = 4, PSML_RNN = 5 } psml_model_kind;

typedef struct {
    int32_t kind;             /* psml_model_kind                                             */
    int32_t n_layers;         /* LINREG/LOGREG/SVM: 1; MLP: len(dims)-1; CNN: 3              */
    int64_t dims[8];          /* MLP: layer widths d_0..d_L; LINREG/LOGREG: {784, 1}         */
    int32_t batch;            /* rows per step per pair (128)                                */
    int32_t lr_shift;         /* eta/|B| = 2^-lr_shift (14)                                  */
    int32_t master_frac_bits; /* m = 27 (R14)                                      */
    uint64_t dealer_seed;     /* DESIGN.md R11: data_seed + 2                                */
    uint32_t pair_id;         /* data-parallel pair index (call-id bits 63:56)               */
    int32_t cnn_c, cnn_h, cnn_w, cnn_k, cnn_cout, cnn_hidden, cnn_classes; /* CNN geometry  */
    int32_t fwd_frac_bits[8]; /* per layer f_w (R21): forward weights W = trunc(W^m,
                                 m - f_w), products with W truncated by f_w; 0 = frac_bits.
                                 frac_bits <= f_w <= m.  The CNN config uses {16, 20, 20}.    */
    int32_t compare;          /* secure comparison of ReLU / Eq. 9: 0 = Kogge-Stone A2B chain +
                                 daBit (R9, 1 + log2 l + 1 rounds), 1 = one-round FSS
                                 DCF comparison (R22; material psml_fss_dealer's layout)       */
    int32_t weight_decay_shift; /* 0 = none; else W^m -= trunc(W^m, shift) every update (SVM:
                                   lambda.eta = 2^-16, R24)                        */
    int32_t rnn_steps;        /* RNN: sequence length T (1..254; call-id layers 1..T+1)       */
    int32_t mask_reuse;       /* DESIGN.md R26 (linear / logistic regression, MLP): the backward
                                 products re-use the forward masks of A_l and W_l and one fresh
                                 mask of delta, so the split engine opens delta once per layer
                                 instead of re-opening A^T, W^T and delta twice                */
    int32_t deal_role;        /* DESIGN.md R23: 0 = the dealer (dealer_seed = the dealer seed; every
                                 stream), 1 / 2 = party 0 / 1 dealing for itself (dealer_seed =
                                 that party's seed s_i = psml_dealer_party_seed(dealer seed, i));
                                 the words it cannot derive come in the dealer's bundle
                                 (psml_model_deal_bundle / psml_model_deal_party)              */
    int32_t strong_pairs;     /* SURVEY C16 / DESIGN.md R28 strong scaling. 0 or 1: this pair's
                                 material is its own (pair field = pair_id; weak scaling).
                                 P >= 2: P pairs train on ONE global batch of P * batch rows, this
                                 pair (pair_id < P) on rows [pair_id * batch, (pair_id + 1) * batch):
                                 the forward / input-gradient products, ReLU / Eq. 9 and Hadamard
                                 material is the row-slice of what a single pair would be dealt
                                 for the global batch (pair field 0; the weight masks V global and
                                 shared), the weight-gradient triplets are this pair's own (pair
                                 field pair_id).  The per-party sum of the P pairs' gradient shares
                                 is the global-batch gradient: update with extra_shift = 0.
                                 Requires batch % 8 == 0 (ChaCha20 block-aligned slices), the
                                 fused dealer (psml_options.fused_dealer), kinds LINREG, LOGREG,
                                 MLP, SVM, RNN and mask_reuse = 0.                               */
} psml_model_desc;

psml_status psml_model_create(psml_ctx ctx, const psml_model_desc *desc, psml_model *out);
psml_status psml_model_destroy(psml_model model);
/* Shape of layer `layer`'s weight matrix (rows x cols). */
psml_status psml_model_layer_shape(psml_model model, int32_t layer, int64_t *rows,
                                   int64_t *cols);
/* Load master-weight shares (m fractional bits) of a layer; the forward copy is
 * W_i = trunc_i(Wm_i, m - f_w) (f_w = fwd_frac_bits[layer], R21).  Wm[i]: device, rows x cols. */
psml_status psml_model_set_master(psml_model model, int32_t layer, const void *const Wm[2],
                                  psml_stream stream);
psml_status psml_model_get_master(psml_model model, int32_t layer, void *const Wm[2],
                                  psml_stream stream);
/* Dealer key separation and compressed distribution (R23).  Party i's material streams
 * are keyed by s_i = psml_dealer_party_seed(dealer_seed, i), so a party regenerates everything it
 * can from s_i alone (party 0: all of its A2B-mode material) and receives only the derived words:
 * party 1's Z_1 of every matrix / conv / Hadamard triplet, c_1 of every boolean AND triplet, r^A_1
 * of every daBit; with the FSS comparison (compare = 1) a party's whole DCF material.
 * psml_model_deal_bundle (a deal_role 0 model): deals `step_id` and gathers party `party`'s derived
 * words into `bundle` (device, caller-owned; NULL = size query) -> *words.
 * psml_model_deal_party (a deal_role 1 + party model): deals its own streams for `step_id` and
 * scatters the bundle over the derived words; the pool is then identical to the dealer's for this
 * party.  Both sides enumerate the words in the same order (items in plan order). */
uint64_t psml_dealer_party_seed(uint64_t dealer_seed, int32_t party);
psml_status psml_model_deal_bundle(psml_model model, uint32_t step_id, int32_t party, void *bundle, int64_t *words,
                                   psml_stream stream);
psml_status psml_model_deal_party(psml_model model, uint32_t step_id, int32_t party, const void *bundle,
                                  int64_t words, psml_stream stream);

/* Offline phase for one step: generate every triplet / MSB material the step's forward and
 * backward pass consumes, with call ids (pair_id, step_id, layer, op, slot) (R11).
 * infer_only = 1 generates only the forward material. */
psml_status psml_model_deal(psml_model model, uint32_t step_id, int32_t infer_only,
                            psml_stream stream);
/* Online phase of one training step on the shares of one minibatch:
 * X[i]: batch x d_0 (CNN: batch x C*H*W), Y[i]: batch x d_L.  Requires psml_model_deal for
 * the same step_id.  Equivalent to forward_backward + apply_update(update_shift = 0). */
psml_status psml_secure_train_step(psml_model model, const void *const X[2],
                                   const void *const Y[2], uint32_t step_id, psml_stream stream);
/* Forward + backward only: leaves the untruncated weight-gradient shares (26 fractional bits)
 * in the model's gradient buffer, for a data-parallel allreduce between pairs. */
psml_status psml_train_forward_backward(psml_model model, const void *const X[2],
                                        const void *const Y[2], uint32_t step_id,
                                        psml_stream stream);
/* Model-owned prediction shares of the last forward pass: yhat[i] is batch x d_L (device). */
psml_status psml_model_output(psml_model model, void **yhat0, void **yhat1, int64_t *n);
/* Contiguous gradient buffer: [party][all layers' rows*cols] words (device, model-owned). */
psml_status psml_model_grads(psml_model model, void **grads, int64_t *words_per_party);
/* W^m_i -= trunc_i(gradW_i, 2f + lr_shift - m + extra_shift); W_i = trunc_i(W^m_i, m - f_w).
 * extra_shift = log2(number of data-parallel pairs summed into the gradient). */
psml_status psml_train_apply_update(psml_model model, int32_t extra_shift, psml_stream stream);
/* CUDA-graph fast path.  Capture ONE training step on `stream` (must not be the legacy default
 * stream) reading the minibatch shares from the fixed device buffers X[2], Y[2]: flags bit 0 =
 * include the dealer (offline material), bit 1 = include the update, bit 2 = PIPELINED dealer:
 * the dealer pools are double-buffered (step s reads pool s % 2) and the graph of step s runs the
 * dealer of step s + 1 on a forked stream concurrently with the online phase of step s (the first
 * step's pool must be filled with psml_model_deal).  The dealer's call ids take their step field
 * from a model-owned device word, so the same graph(s) serve every step.
 * Without bit 0 the graph consumes material dealt by psml_model_deal for exactly the replayed
 * step id (one graph per pool), once: dealer material is single-use (a mask opened on two values
 * leaks their difference), and the eager calls consume it the same way.  Bit 3 (only without
 * bits 0 and 2) = UNSAFE benchmark-only replay of pool 0 as last dealt, for timing the online
 * phase alone; never used for training.
 * psml_model_step_graph writes the step word and launches the graph; the caller refills X/Y
 * before each replay; pipelined steps must be consecutive (PSML_ERR_STATE otherwise).
 * Capture must not overlap other work on the stream. */
psml_status psml_model_capture_step(psml_model model, const void *const X[2], const void *const Y[2],
                                    int32_t flags, psml_stream stream);
psml_status psml_model_step_graph(psml_model model, uint32_t step_id, psml_stream stream);
/* One whole step from HOST buffers (the client's end-to-end call): copies the
 * minibatch's 8-bit pixels q (batch x d_0 bytes, host; pinned memory makes the copies
 * asynchronous) and its labels y (y_kind 0: float64 batch x d_L; 1: uint8 class indices of one-hot
 * labels, batch bytes) to model-owned device staging, encodes and shares them into the captured
 * X/Y buffers (psml_encode_share_u8 / _onehot / psml_encode_share, share ids = call id
 * (pair, step_id, 0, op 7, slot 0/1) under share_seed; R11), replays the captured step
 * (psml_model_step_graph, same preconditions) and copies both parties' prediction shares
 * (2 x batch x d_L words, party 0 first) to yhat_host (host).  Asynchronous on `stream`: the
 * host buffers must stay valid until it completes.  PSML_ERR_STATE without a captured step. */
psml_status psml_model_step_host(psml_model model, const uint8_t *q, const void *y, int32_t y_kind,
                                 uint64_t share_seed, uint32_t step_id, void *yhat_host, psml_stream stream);
/* One whole step from DEVICE plaintext (the client's batch already in HBM): encodes and shares
 * X (batch x features float64, device) and Y (batch x d_L float64, device) into the captured X/Y
 * buffers in ONE launch -- bit-identical to psml_encode_share with the share ids of
 * psml_model_step_host -- then replays the captured step (psml_model_step_graph, same
 * preconditions).  Co-resident captured step only; asynchronous on `stream`. */
psml_status psml_model_step_device(psml_model model, const double *X, const double *Y, uint64_t share_seed,
                                   uint32_t step_id, psml_stream stream);
/* Number of kernel nodes in the captured step graph (launch accounting for bench.py). */
psml_status psml_model_graph_nodes(psml_model model, int64_t *n);
/* Secure inference (the forward half): Yhat[i]: batch x d_L.  Needs
 * psml_model_deal(step_id, infer_only=1) (or a full deal) for the same step_id. */
psml_status psml_secure_infer(psml_model model, const void *const X[2], uint32_t step_id,
                              void *const Yhat[2], psml_stream stream);

/* ------------------------------------------------------------------------------------------ */
/* Split deployment: ONE party per process / GPU (Fig. 1b L55-L61: two non-colluding  */
/* servers; L65 "compute E and F via communication").  Every opening of the training step --   */
/* the E/F of each Beaver product (Eq. 5), the boolean AND rounds of the MSB chain, the daBit  */
/* B2A word and the Hadamard E/F (R9) -- becomes one symmetric exchange of the        */
/* party's masked message through a transport.  Shares and opened values are bit-identical to */
/* the co-resident engine (same kernels, restricted to one party).                              */
/* ------------------------------------------------------------------------------------------ */
typedef struct psml_xport_s *psml_xport;

/* Host callback transport (any backend; used for host-staged gloo).  Must send, for every
 * k < n, `bytes[k]` bytes at device address send[k] to the peer and receive the peer's
 * same-sized message into device address recv[k], ordered after the work already enqueued on
 * `stream` and before work enqueued after it returns (synchronise the stream first).  Returns 0
 * on success; non-zero makes the step fail with PSML_ERR_NCCL. */
typedef int32_t (*psml_exchange_fn)(void *user, int32_t n, void *const *send, void *const *recv,
                                    const int64_t *bytes, psml_stream stream);

/* 128-byte NCCL unique id (created by one party, broadcast by the caller, e.g. over a
 * torch.distributed process group). */
psml_status psml_nccl_unique_id(uint8_t uid[128]);
/* NCCL transport: the library creates and owns a 2-rank communicator (this party = `rank`,
 * the peer = 1 - rank) on the current device; exchanges are grouped ncclSend/ncclRecv on the
 * step's stream (stream-ordered, no host synchronisation; NVLink P2P between GPUs). */
psml_status psml_xport_nccl_create(const uint8_t uid[128], int32_t rank, psml_xport *out);
psml_status psml_xport_callback_create(psml_exchange_fn fn, void *user, psml_xport *out);
/* Peer-memory transport (the B200-native one).  Each party allocates a
 * double-buffered mailbox of 2 x capacity_bytes (+ a few flag words) in its own HBM and exports
 * a PSML_PEER_HANDLE_BYTES blob (CUDA IPC handles + process id); the caller ships the blob to the
 * peer (e.g. all_gather over a torch.distributed group) and both call psml_xport_peer_connect
 * with the other party's blob.  The peer's mailbox is then mapped into this process (CUDA IPC:
 * NVLink P2P between two GPUs, the same HBM for two processes on one GPU; a raw pointer when
 * both parties live in one process).  One exchange is ONE kernel on the caller's stream: it
 * stores this party's messages into the peer's mailbox, releases a sequence number into the
 * peer's flag word (system scope), waits for the peer's, and copies its own mailbox out to
 * `recv` -- no host synchronisation, and graph-capturable (sequence numbers live in device
 * memory).  An exchange larger than capacity_bytes runs as several mailbox rounds.  Both
 * parties must issue the same exchanges in the same order (like NCCL collectives); a peer that
 * stops answering makes the kernel trap after 60 s (PSML_ERR_CUDA on the next call) instead of
 * hanging the GPU.  party: 0 or 1; capacity_bytes >= 4096, equal on both sides. */
#define PSML_PEER_HANDLE_BYTES 256
psml_status psml_xport_peer_create(int32_t party, int64_t capacity_bytes, psml_xport *out,
                                   uint8_t handle[PSML_PEER_HANDLE_BYTES]);
psml_status psml_xport_peer_connect(psml_xport x, const uint8_t peer_handle[PSML_PEER_HANDLE_BYTES]);
psml_status psml_xport_destroy(psml_xport x);
/* One symmetric exchange of n device buffers (what every opening round does). */
psml_status psml_xport_exchange(psml_xport x, int32_t n, const void *const *send, void *const *recv,
                                const int64_t *bytes, psml_stream stream);
/* Bytes and exchanges issued through this transport so far (accounting for bench.py). */
psml_status psml_xport_stats(psml_xport x, int64_t *bytes_sent, int64_t *exchanges);

/* Data-parallel communicator of ONE party over its `size` GPUs (pair k = ranks k
 * and k + N/2; party i's N/2 GPUs sum their untruncated gradient shares).  Library-owned NCCL
 * communicator built from a 128-byte unique id (psml_nccl_unique_id on rank 0 of the party,
 * broadcast by the caller); size 1 needs no id (uid may be NULL) and makes the all-reduce a no-op.
 * psml_dp_allreduce: in-place sum of n ring words (uint64_t for l = 64, uint32_t for l = 32) over
 * the party's ranks = addition in Z_{2^l} (ncclSum on unsigned words wraps), stream-ordered and
 * graph-capturable. */
typedef struct psml_dp_s *psml_dp;
psml_status psml_dp_create(const uint8_t uid[128], int32_t rank, int32_t size, psml_dp *out);
psml_status psml_dp_destroy(psml_dp dp);
psml_status psml_dp_size(psml_dp dp, int32_t *size);
psml_status psml_dp_allreduce(psml_dp dp, void *buf, int64_t n, int32_t l, psml_stream stream);

/* Per-party context (one ctx per party per GPU per process).  The context carries
 * this party, its pair transport (psml_xport_*_create, caller-owned, must outlive the ctx) and
 * its data-parallel communicator (nullable).  psml_secure_matmul_party is the collective
 * one-party Beaver product: both parties call it with identical shapes and flags in the same
 * order; it masks E_i = op(A)_i - U_i, F_i = op(B)_i - V_i (Eq. 4), exchanges them through the
 * pair transport (Eq. 5), and computes C_i = i.E.F + E.V_i + U_i.F + Z_i (Eq. 8 shape) with
 * SecureML truncation by trunc_bits -- bit-identical to psml_secure_matmul's party-i share.
 * All pointers are this party's device buffers; flags: PSML_TRANS_A / PSML_TRANS_B. */
psml_status psml_ctx_create_party(psml_ring ring, int32_t gemm_backend, int32_t party, psml_xport pair, psml_dp dp,
                                  psml_ctx *out);
psml_status psml_secure_matmul_party(psml_ctx ctx, const void *A_i, const void *B_i, const void *U_i, const void *V_i,
                                     const void *Z_i, int64_t M, int64_t K, int64_t N, int32_t flags,
                                     int32_t trunc_bits, void *C_i, psml_stream stream);

/* Party `party`'s half of one training step (LINREG / LOGREG / MLP / CNN): X_i: batch x d_0
 * (CNN: batch x C*H*W), Y_i: batch x d_L, this party's shares (device).  The model's dealer
 * pool must hold the step's material (psml_model_deal; in this simulation each party's process
 * runs the dealer and reads only its own half -- a deployment ships it from the client).
 * Leaves this party's untruncated weight-gradient share in psml_model_grads()[party] and its
 * prediction share in psml_model_output; then psml_party_apply_update updates this party's
 * master/forward weight shares (extra_shift as psml_train_apply_update).  Both parties must
 * call with the same step_id; every exchange is collective between them. */
psml_status psml_party_forward_backward(psml_model model, int32_t party, psml_xport x,
                                        const void *X_i, const void *Y_i, uint32_t step_id,
                                        psml_stream stream);
psml_status psml_party_apply_update(psml_model model, int32_t party, int32_t extra_shift,
                                    psml_stream stream);
/* The whole step of one party: psml_party_forward_backward, then psml_dp_allreduce of this
 * party's gradient share over `dp` (nullable = one pair), then psml_party_apply_update with
 * extra_shift = log2(dp size) (the size must be a power of two). */
psml_status psml_party_train_step(psml_model model, int32_t party, psml_xport x, psml_dp dp, const void *X_i,
                                  const void *Y_i, uint32_t step_id, psml_stream stream);
/* CUDA-graph capture of psml_party_train_step (same flags as psml_model_capture_step: bit 0 the
 * dealer in the graph, bit 1 the update (and the all-reduce), bit 2 pipelined dealer); replay with
 * psml_model_step_graph.  The transport must be graph-capturable (peer memory or NCCL, not a host
 * callback: PSML_ERR_UNSUPPORTED).  Both parties capture and replay the same step sequence. */
psml_status psml_party_capture_step(psml_model model, int32_t party, psml_xport x, psml_dp dp, const void *X_i,
                                    const void *Y_i, int32_t flags, psml_stream stream);

#ifdef __cplusplus
}
#endif
#endif /* PSML_H_ */
