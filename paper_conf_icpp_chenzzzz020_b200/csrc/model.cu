// model.cu -- secure training / inference of linear & logistic regression, MLP and CNN on the
// co-resident pair engine (Sec. 4.3 "Detailed Design" L201-L207; Sec. 7.1).
//
// One step (per pair, batch B rows), all in Z_{2^64} with f = 13 fractional bits:
//   forward   z_l = trunc(h_l . W_l)            Beaver matmul (op 0)
//             h_{l+1} = ReLU(z_l)  (hidden)      MSB chain + Hadamard (ops 3, 6/0), keeps DReLU
//             yhat = Eq. 9(z_L) (logistic/MLP/CNN) or z_L (linear)   (ops 4, 6/2)
//   backward  delta = yhat - y
//             gW_l = h_l^T . delta               Beaver matmul, untruncated (op 1)
//             delta = trunc(delta . W_l^T) (.) DReLU_{l-1}   (op 2, Hadamard 6/1)
//   update    W^m_l -= trunc(gW_l, 26 + s_lr - m); W_l = trunc(W^m_l, m - f)   (R14)
// Every triplet / MSB material comes from the model's dealer pool filled by psml_model_deal with
// call id (pair, step, layer, op, slot) -- identical to oracle/protocol.py (R11).
#include <cstring>
#include <memory>
#include <string>
#include <vector>

#include "engine.h"
#include "dealer_fused.cuh"
#include "fused.cuh"
#include "fss.cuh"
#include "split_fused.cuh"

namespace psml {

using T = uint64_t;

enum { OP_FWD = 0, OP_GRADW = 1, OP_GRADIN = 2, OP_RELU_MSB = 3, OP_EQ9_MSB = 4, OP_HADAMARD = 6, OP_SHARE = 7 };
enum ItemKind { IT_MATRIX, IT_CONV_FWD, IT_CONV_GW, IT_HAD, IT_MSB, IT_FSS };   // IT_FSS: DCF material (R22)

__global__ void set_word_kernel(uint32_t *p, uint32_t v) { *p = v; }
// last node of a pipelined graph's dealer branch: the next consecutive replay's step word
__global__ void advance_word_kernel(uint32_t *p) { *p += 1; }

// Co-resident Beaver matmuls run the explicit mask round then the GEMM that opens E/F (default:
// measured faster inside the CUDA graph, 338K vs 328K samples/s) or fuse the mask into the GEMM's
// operand loads (psml_options.fused_open: faster eagerly, one launch less); bit-identical (tested).
static bool fused_open() { return cur_opts().fused_open != 0; }

// Fused co-resident training step (fused.cuh): producers open their consumers' operands
// (default) or one open pass per product (psml_options.fused_step = 0); bit-identical (tested).
static bool fuse_enabled() { return cur_opts().fused_step != 0; }

// The whole dealer of one step as two launches (dealer_fused.cuh; default) or one launch group per
// item (psml_options.fused_dealer = 0); bit-identical (tested).
static bool fused_deal() { return cur_opts().fused_dealer != 0; }

static inline uint64_t call_id(uint32_t pair, uint32_t step, int layer, int op, int slot) {
    return ((uint64_t)(pair & 0xFF) << 56) | ((uint64_t)step << 24) | ((uint64_t)(layer & 0xFF) << 16) |
           ((uint64_t)(op & 0xFF) << 8) | (uint64_t)(slot & 0xFF);
}

struct Buf {  // a pair of device buffers of `n` words
    T *p[2] = {nullptr, nullptr};
    int64_t n = 0;
    T *const *pp() { return p; }
    const T *const *cp() const { return (const T *const *)p; }
};

struct DealItem {
    ItemKind kind;
    int layer, op, slot;
    int64_t M = 0, K = 0, N = 0, n = 0;
    bool fwd = true;  // needed by inference
    Buf U, V, Z, mat;
};

struct OpenBuf {    // opened operands of one matrix product (fused step): E, X_1 (M x K), F (K x N)
    T *E = nullptr, *X1 = nullptr, *F = nullptr;
};

struct DealPlan {   // fused dealer of one pool (full or inference-only)
    PrgJob *prg = nullptr;
    int n_prg = 0;
    int64_t prg_blocks = 0;
    int n_prg_mat = 0;           // jobs [0, n_prg_mat) = matrix-triplet streams (U, V, Z_0), needed
    int64_t prg_mat_blocks = 0;  // by the Z = U V launch; the rest (AND/daBit/Hadamard) after them
    double chacha_blocks = 0;   // ChaCha20 block evaluations of the PRG work list (all streams)
    ClJob<DealerOps<T>> *gemm = nullptr;
    int n_gemm = 0, gemm_ks = 4;
    bool gemm_big = false;   // 64 x 64 tiles, 4 x 4 per thread (ClDealer) instead of ClDefault
    int64_t gemm_tiles = 0;
    std::vector<int> rest;   // items whose Z = U V runs in its own launch (conv, tcgen05-sized)
    std::vector<int> fss;    // DCF key generation (own launch per item, R22)
};

}  // namespace psml

struct psml_model_s {
    psml::Ctx *ctx = nullptr;
    psml_model_desc d{};
    int nl = 0;
    int64_t B = 0;
    std::vector<int64_t> rows, cols;  // weight shapes
    std::vector<int64_t> dims;        // MLP-style widths d_0..d_L (CNN: d_1 = 12544 after conv)
    psml::ConvGeom g{};
    std::vector<psml::Buf> Wm, W;
    psml::T *grad_base = nullptr;
    int64_t grad_words = 0;
    std::vector<int64_t> grad_off;
    // activations
    std::vector<psml::Buf> act, z, drelu;  // act[l]: input of layer l (l >= 1 model-owned)
    psml::Buf yhat, delta, tmp;
    // Dealer pools, double-buffered: step s consumes pool s % 2, so the dealer of step s + 1 can
    // run concurrently with the online phase of step s (offline/online pipelining).
    std::vector<psml::DealItem> items[2];
    psml::DealPlan plan[2][2];         // [pool][infer_only]
    std::vector<psml::OpenBuf> ob;     // per item index (fused step; empty when not eligible)
    int pool = 0;                      // pool the online phase is reading
    psml::T *ws = nullptr;             // online workspace
    int64_t ws_words = 0;
    psml::T *dws = nullptr;            // dealer workspace (split-K partials of Z = U V)
    int64_t dws_words = 0;
    std::vector<void *> allocs;
    int64_t dealt_step[2] = {-1, -1};
    bool dealt_full[2] = {false, false};
    bool grads_ready = false;
    uint32_t *step_dev = nullptr;      // device copy of the step number (dealer call ids)
    int64_t word_next = -1;            // value *step_dev holds once the last enqueued pipelined
                                       // replay completes (it advances the word itself); -1 unknown
    cudaGraphExec_t graph[2] = {nullptr, nullptr};  // captured step(s) (psml_model_capture_step)
    cudaGraph_t graph_tmpl[2] = {nullptr, nullptr};  // their templates (the share node's handle lives there)
    cudaGraphNode_t share_node[2] = {nullptr, nullptr};   // the client's encode + share, first online node
    bool share_live[2] = {false, false};              // the node holds a real batch's job (else a no-op)
    // the client's read-back of both prediction shares (psml_model_step_host into mapped pinned
    // memory) as a graph node on its own branch, forked as soon as the forward pass wrote them
    cudaGraphNode_t out_node[2] = {nullptr, nullptr};
    bool out_live[2] = {false, false};
    bool cap_out = false;              // (capture) fork the read-back branch after the forward pass
    cudaStream_t d2h = nullptr;
    cudaEvent_t ev_y = nullptr, ev_yj = nullptr;
    unsigned share_grid = 0;
    int graph_flags = 0;
    int64_t graph_kernels = 0;
    cudaStream_t side = nullptr;       // dealer branch inside the pipelined graph
    cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
    cudaStream_t hi = nullptr;         // online phase inside the pipelined graph (highest priority)
    cudaEvent_t ev_hi = nullptr;
    cudaEvent_t ev_late = nullptr;
    const void *cap_X[2] = {nullptr, nullptr}, *cap_Y[2] = {nullptr, nullptr};   // captured step inputs
    uint8_t *stage_q = nullptr;        // device staging of psml_model_step_host (pixels, labels)
    void *stage_y = nullptr;
    cudaStream_t gw = nullptr;         // weight-gradient branch of the backward pass (highest priority)
    cudaEvent_t ev_gw = nullptr, ev_gwj = nullptr;
    cudaStream_t side2 = nullptr;      // second dealer branch (AND / daBit / Hadamard PRG streams)
    cudaEvent_t ev_d2 = nullptr, ev_d2j = nullptr;     // late fork point of the dealer branch (PSML_DEAL_AFTER)
    int deal_pending_pool = -1;        // capture in progress: dealer branch not forked yet
    int deal_after = 0, deal_stage = 0;
    bool deal_alone = false;           // dealer being captured after the online chain (full PRG grid)
    bool deal_on_launch = false;       // fork the dealer at the first product's launch completion
    bool fork_event_armed = false;     // ev_late is that launch's completion event
    // split deployment capture (psml_party_capture_step): the party, its pair transport and its
    // data-parallel communicator; cap_party < 0 = the co-resident engine
    int cap_party = -1;
    psml::DealSeeds seeds{};           // dealer key separation (R23), from dealer_seed and deal_role
    // RNN (R25): per time step inputs A_t = [x_t | h_{t-1}], states h_t, DReLU_t, and the
    // per-step weight-gradient product before it is added into the layer-0 gradient
    psml::Buf rnnA, rnnH, rnnD, rnnG;
    // split engine with mask reuse (R26): this party's copy of each layer's forward openings E, F,
    // the opened delta, and scratch (transposes, a zero operand, delta's send / receive messages)
    std::vector<psml::T *> eopen, fopen;
    psml::T *dopen = nullptr, *rT = nullptr, *rzero = nullptr, *dms = nullptr, *dmr = nullptr;
    int rnn_T = 0, rnn_D = 0;
    psml_xport cap_xport = nullptr;
    psml_dp cap_dp = nullptr;
};

namespace psml {

static psml_status dalloc(psml_model_s *m, T **out, int64_t words) {
    if (words <= 0) { *out = nullptr; return PSML_OK; }
    void *p = nullptr;
    if (cudaMalloc(&p, sizeof(T) * (size_t)words) != cudaSuccess) {
        cudaGetLastError();
        return fail(PSML_ERR_NOMEM, "model allocation of " + std::to_string(words * 8) + " bytes failed");
    }
    m->allocs.push_back(p);
    *out = (T *)p;
    return PSML_OK;
}

static psml_status balloc(psml_model_s *m, Buf &b, int64_t n) {
    b.n = n;
    PSML_TRY(dalloc(m, &b.p[0], n));
    return dalloc(m, &b.p[1], n);
}

static DealItem *find_item(psml_model_s *m, int layer, int op, int slot) {
    for (auto &it : m->items[m->pool])
        if (it.layer == layer && it.op == op && it.slot == slot) return &it;
    return nullptr;
}

static void add_matrix(psml_model_s *m, int layer, int op, int64_t M, int64_t K, int64_t N, bool fwd) {
    DealItem it;
    it.kind = IT_MATRIX; it.layer = layer; it.op = op; it.slot = 0; it.M = M; it.K = K; it.N = N; it.fwd = fwd;
    m->items[0].push_back(it);
}
static void add_had(psml_model_s *m, int layer, int slot, int64_t n, bool fwd) {
    DealItem it;
    it.kind = IT_HAD; it.layer = layer; it.op = OP_HADAMARD; it.slot = slot; it.n = n; it.fwd = fwd;
    m->items[0].push_back(it);
}
static void add_msb(psml_model_s *m, int layer, int op, int64_t n, bool fwd) {
    DealItem it;
    it.kind = m->d.compare == 1 ? IT_FSS : IT_MSB;   // comparison material: A2B chain (R9) or DCF (R22)
    it.layer = layer; it.op = op; it.slot = 0; it.n = n; it.fwd = fwd;
    m->items[0].push_back(it);
}

// Strong-scaling view of a dealer item (R28): with strong_pairs = P > 1
// every item whose output rows are batch rows is the row-slice of the material a single pair
// would be dealt for the global batch (pair field 0, stream elements offset by the slice start);
// the weight-gradient triplets (contractions over the batch) stay this pair's own.
static bool strong_rows(const psml_model_s *m, const DealItem &it) {
    return m->d.strong_pairs > 1 && !(it.kind == IT_MATRIX && it.op == OP_GRADW);
}
static uint32_t item_pair(const psml_model_s *m, const DealItem &it) { return strong_rows(m, it) ? 0u : m->d.pair_id; }
// row-ordered parts of an elementwise item: Eq. 9's [z + 1/2 ; z - 1/2] material is 2 parts, so a
// pair's slice is one range in each half of the global layout
static int item_parts(const DealItem &it) {
    const bool eq9 = ((it.kind == IT_MSB || it.kind == IT_FSS) && it.op == OP_EQ9_MSB) || (it.kind == IT_HAD && it.slot == 2);
    return eq9 ? 2 : 1;
}
// stream element of local element h * per of part h (per = n / parts elements per part)
static int64_t strong_elem0(const psml_model_s *m, int64_t per, int h) {
    return ((int64_t)h * m->d.strong_pairs + m->d.pair_id) * per;
}

static bool is_eq9_out(const psml_model_s *m) { return m->d.kind != PSML_LINREG && m->d.kind != PSML_SVM; }
// forward-weight fractional bits of layer l (R21)
static int fw(const psml_model_s *m, int l) {
    const int v = m->d.fwd_frac_bits[l];
    return v > 0 ? v : m->ctx->ring.frac_bits;
}

static void plan_items(psml_model_s *m) {
    const int64_t B = m->B;
    if (m->d.kind == PSML_CNN) {
        const ConvGeom &g = m->g;
        const int64_t rows = B * g.OH * g.OW, kk = (int64_t)g.C * g.k * g.k;
        const int64_t h1 = m->dims[1], hid = m->dims[2], cls = m->dims[3];
        DealItem cf;
        cf.kind = IT_CONV_FWD; cf.layer = 0; cf.op = OP_FWD; cf.slot = 0;
        cf.M = rows; cf.K = kk; cf.N = m->cols[0]; cf.fwd = true;
        m->items[0].push_back(cf);
        add_msb(m, 0, OP_RELU_MSB, B * h1, true);
        add_had(m, 0, 0, B * h1, true);
        add_matrix(m, 1, OP_FWD, B, h1, hid, true);
        add_msb(m, 1, OP_RELU_MSB, B * hid, true);
        add_had(m, 1, 0, B * hid, true);
        add_matrix(m, 2, OP_FWD, B, hid, cls, true);
        add_msb(m, 2, OP_EQ9_MSB, 2 * B * cls, true);
        add_had(m, 2, 2, 2 * B * cls, true);
        add_matrix(m, 2, OP_GRADW, hid, B, cls, false);
        add_matrix(m, 2, OP_GRADIN, B, cls, hid, false);
        add_had(m, 1, 1, B * hid, false);
        add_matrix(m, 1, OP_GRADW, h1, B, hid, false);
        add_matrix(m, 1, OP_GRADIN, B, hid, h1, false);
        add_had(m, 0, 1, B * h1, false);
        DealItem cg;
        cg.kind = IT_CONV_GW; cg.layer = 0; cg.op = OP_GRADW; cg.slot = 0;
        cg.M = kk; cg.K = rows; cg.N = m->cols[0]; cg.fwd = false;
        m->items[0].push_back(cg);
        return;
    }
    if (m->d.kind == PSML_RNN) {   // Elman RNN, backpropagation through time (R25)
        const int T = m->rnn_T;
        const int64_t K1 = m->rows[0], H = m->dims[1], C = m->dims[2];
        for (int t = 1; t <= T; ++t) {
            add_matrix(m, t, OP_FWD, B, K1, H, true);
            add_msb(m, t, OP_RELU_MSB, B * H, true);
            add_had(m, t, 0, B * H, true);
        }
        add_matrix(m, T + 1, OP_FWD, B, H, C, true);
        add_msb(m, T + 1, OP_EQ9_MSB, 2 * B * C, true);
        add_had(m, T + 1, 2, 2 * B * C, true);
        add_matrix(m, T + 1, OP_GRADW, H, B, C, false);
        add_matrix(m, T + 1, OP_GRADIN, B, C, H, false);
        add_had(m, T, 1, B * H, false);
        for (int t = T; t >= 1; --t) {
            add_matrix(m, t, OP_GRADW, K1, B, H, false);
            if (t > 1) {
                add_matrix(m, t, OP_GRADIN, B, H, H, false);
                add_had(m, t - 1, 1, B * H, false);
            }
        }
        return;
    }
    if (m->d.kind == PSML_SVM) {   // linear SVM, hinge subgradient (R24)
        add_matrix(m, 0, OP_FWD, B, m->dims[0], 1, true);
        add_had(m, 0, 3, B, false);                 // margin y (.) z
        add_msb(m, 0, OP_RELU_MSB, B, false);       // [y z - 1 < 0]
        add_had(m, 0, 4, B, false);                 // y (.) ind
        add_matrix(m, 0, OP_GRADW, m->dims[0], B, 1, false);
        return;
    }
    const int nl = m->nl;
    for (int l = 0; l < nl; ++l) {
        add_matrix(m, l, OP_FWD, B, m->dims[l], m->dims[l + 1], true);
        const int64_t n = B * m->dims[l + 1];
        if (l < nl - 1) {
            add_msb(m, l, OP_RELU_MSB, n, true);
            add_had(m, l, 0, n, true);
        } else if (is_eq9_out(m)) {
            add_msb(m, l, OP_EQ9_MSB, 2 * n, true);
            add_had(m, l, 2, 2 * n, true);
        }
    }
    for (int l = nl - 1; l >= 0; --l) {
        add_matrix(m, l, OP_GRADW, m->dims[l], B, m->dims[l + 1], false);
        if (l > 0) {
            add_matrix(m, l, OP_GRADIN, B, m->dims[l + 1], m->dims[l], false);
            add_had(m, l - 1, 1, B * m->dims[l], false);
        }
    }
}

static psml_status alloc_items(psml_model_s *m, std::vector<DealItem> &items) {
    const psml_ring ring = m->ctx->ring;
    for (auto &it : items) {
        switch (it.kind) {
        case IT_MATRIX:
            PSML_TRY(balloc(m, it.U, it.M * it.K));
            PSML_TRY(balloc(m, it.V, it.K * it.N));
            PSML_TRY(balloc(m, it.Z, it.M * it.N));
            break;
        case IT_CONV_FWD:
        case IT_CONV_GW: {
            const int64_t nin = m->B * m->g.C * m->g.H * m->g.W;
            PSML_TRY(balloc(m, it.U, nin));
            PSML_TRY(balloc(m, it.V, it.K * it.N));
            PSML_TRY(balloc(m, it.Z, it.M * it.N));
            break;
        }
        case IT_HAD:
            PSML_TRY(balloc(m, it.U, it.n));
            PSML_TRY(balloc(m, it.V, it.n));
            PSML_TRY(balloc(m, it.Z, it.n));
            break;
        case IT_MSB:
            PSML_TRY(balloc(m, it.mat, psml_msb_material_words(ring, it.n)));
            break;
        case IT_FSS:
            PSML_TRY(balloc(m, it.mat, (int64_t)FSS_WORDS * it.n));
            break;
        }
    }
    return PSML_OK;
}

static int64_t ws_need(psml_model_s *m) {
    int64_t w = 0;
    for (auto &it : m->items[0]) {
        switch (it.kind) {
        case IT_MATRIX:
            w = std::max(w, beaver_ws_words<T>(it.M, it.K, it.N));
            if (m->ctx->use_tc(it.M, 2 * it.K, it.N))
                w = std::max(w, (int64_t)(tc_beaver_ws_bytes<T>(it.M, it.K, it.N) + 7) / 8);
            break;
        case IT_CONV_FWD: w = std::max(w, conv_ws_words<T>(m->B, m->g, 0, it.N)); break;
        case IT_CONV_GW: w = std::max(w, conv_ws_words<T>(m->B, m->g, 1, it.N)); break;
        case IT_HAD: w = std::max(w, 4 * it.n); break;
        case IT_MSB: w = std::max(w, msb_ws_words<T>(it.n)); break;
        case IT_FSS: w = std::max(w, 12 * it.n); break;
        }
    }
    return w;
}

static int64_t dws_need(psml_model_s *m) {
    int64_t w = 1;   // dealer: split-K partials of the Z = U V GEMMs (or the tcgen05 limb planes)
    for (auto &it : m->items[0]) {
        if (it.kind != IT_HAD && it.kind != IT_MSB && it.kind != IT_FSS) w = std::max(w, it.M * it.N);
        if (it.kind == IT_MATRIX && m->ctx->use_tc(it.M, it.K, it.N))
            w = std::max(w, (int64_t)(tc_ring_gemm_ws_bytes(64, it.M, it.K, it.N) + 7) / 8);
    }
    return w;
}

// ------------------------------------------------------------------------------------------------
// dealer (offline phase)
// ------------------------------------------------------------------------------------------------
// PRG part of a matrix / conv triplet: U_0, U_1 (n_u), V_0, V_1 (K x N), Z_0 (M x N)
static psml_status deal_prg(psml_model_s *m, DealItem &it, uint64_t cid, cudaStream_t s) {
    const DealSeeds &S = m->seeds;
    ProfScope prof(PROF_DEALER, s, (double)sizeof(T) * (2 * it.U.n + 2 * it.V.n + it.Z.n));
    dealer_pair_kernel<T><<<grid_for(it.U.n / 8 + 1, 256), 256, 0, s>>>(
        dkey(S, TAG_U0, cid, m->step_dev), dkey(S, TAG_U1, cid, m->step_dev), it.U.n, it.U.p[0],
        it.U.p[1], nullptr);
    PSML_LAUNCH_CHECK();
    dealer_pair_kernel<T><<<grid_for(it.V.n / 8 + 1, 256), 256, 0, s>>>(
        dkey(S, TAG_V0, cid, m->step_dev), dkey(S, TAG_V1, cid, m->step_dev), it.V.n, it.V.p[0],
        it.V.p[1], nullptr);
    PSML_LAUNCH_CHECK();
    prg_kernel<T, 0><<<grid_for(it.Z.n / 8 + 2, 256), 256, 0, s>>>(dkey(S, TAG_Z0, cid, m->step_dev), 0, it.Z.n,
                                                                     it.Z.p[0], nullptr, nullptr);
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

// Z = U V part of a matrix / conv triplet (after its PRG part)
static psml_status deal_gemm(psml_model_s *m, DealItem &it, cudaStream_t s) {
    if (it.kind == IT_MATRIX) {
        if (m->ctx->use_tc(it.M, it.K, it.N))
            return tc_dealer_gemm(64, it.U.p[0], it.U.p[1], it.V.p[0], it.V.p[1], it.M, it.K, it.N, it.Z.p[0],
                                  it.Z.p[1], m->dws, sizeof(T) * (size_t)m->dws_words, s);
        DealerOps<T> ops;   // Z_1 = (U_0 + U_1)(V_0 + V_1) - Z_0
        ops.U0 = it.U.p[0]; ops.U1 = it.U.p[1]; ops.V0 = it.V.p[0]; ops.V1 = it.V.p[1];
        ops.Z0 = it.Z.p[0]; ops.Z1 = it.Z.p[1];
        ops.M = it.M; ops.N = it.N; ops.Kext = it.K;
        return launch_ring_gemm<T, DealerOps<T>>(ops, m->dws, m->dws_words, s, m->ctx->sm_count);
    }
    ConvDealerOps<T> ops;   // Z_1 = im2col(U_0 + U_1) (^T) (V_0 + V_1) - Z_0
    ops.U0 = it.U.p[0]; ops.U1 = it.U.p[1]; ops.V0 = it.V.p[0]; ops.V1 = it.V.p[1];
    ops.Z0 = it.Z.p[0]; ops.Z1 = it.Z.p[1];
    ops.g = m->g; ops.M = it.M; ops.N = it.N; ops.Kext = it.K; ops.transposed = it.kind == IT_CONV_GW;
    return launch_ring_gemm<T, ConvDealerOps<T>>(ops, m->dws, m->dws_words, s, m->ctx->sm_count);
}

// out_p = transpose(in_p): in is R x C row-major, out C x R (both parties)
static __global__ void transpose_pair_kernel(CPair<T> in, int64_t R, int64_t C, Pair<T> out) {
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < R * C; e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = e / C, c = e % C;
#pragma unroll
        for (int p = 0; p < 2; ++p) out.p[p][c * R + r] = in.p[p][e];
    }
}

// SecureML mask reuse (R26): the backward triplets of layer l copy the forward masks --
// gradW: U = U_f^T, V = D;  gradin: U = D, V = V_f^T -- with D = PRG("U0"/"U1") under the gradin
// call id; Z_0 = PRG("Z0") under the item's own call id and Z_1 = U V - Z_0 as usual.
static psml_status deal_reuse_item(psml_model_s *m, DealItem &it, uint32_t step, cudaStream_t s) {
    DealItem *f = nullptr;   // the forward triplet of the same layer in the same pool as `it`
    for (auto &items : m->items)
        if (&it >= items.data() && &it < items.data() + items.size())
            for (auto &x : items)
                if (x.layer == it.layer && x.op == OP_FWD && x.kind == IT_MATRIX) f = &x;
    if (!f) return fail(PSML_ERR_STATE, "mask reuse: missing forward triplet");
    const DealSeeds &S = m->seeds;
    const uint64_t cgi = call_id(m->d.pair_id, step, it.layer, OP_GRADIN, 0);
    const uint64_t cid = call_id(m->d.pair_id, step, it.layer, it.op, it.slot);
    const int64_t B = f->M, din = f->K, dout = f->N;
    Buf &D = it.op == OP_GRADW ? it.V : it.U;   // B x dout
    dealer_pair_kernel<T><<<grid_for(D.n / 8 + 1, 256), 256, 0, s>>>(dkey(S, TAG_U0, cgi, m->step_dev),
                                                                     dkey(S, TAG_U1, cgi, m->step_dev), D.n, D.p[0],
                                                                     D.p[1], nullptr);
    PSML_LAUNCH_CHECK();
    if (it.op == OP_GRADW)   // U = U_f^T (din x B)
        transpose_pair_kernel<<<ew_grid(B * din), EW_THREADS, 0, s>>>(CPair<T>{{f->U.p[0], f->U.p[1]}}, B, din,
                                                                      Pair<T>{{it.U.p[0], it.U.p[1]}});
    else                     // V = V_f^T (dout x din)
        transpose_pair_kernel<<<ew_grid(din * dout), EW_THREADS, 0, s>>>(CPair<T>{{f->V.p[0], f->V.p[1]}}, din, dout,
                                                                         Pair<T>{{it.V.p[0], it.V.p[1]}});
    PSML_LAUNCH_CHECK();
    prg_kernel<T, 0><<<grid_for(it.Z.n / 8 + 2, 256), 256, 0, s>>>(dkey(S, TAG_Z0, cid, m->step_dev), 0, it.Z.n,
                                                                     it.Z.p[0], nullptr, nullptr);
    PSML_LAUNCH_CHECK();
    return deal_gemm(m, it, s);
}

static psml_status deal_item(psml_model_s *m, DealItem &it, uint32_t step, cudaStream_t s) {
    const uint64_t seed = m->d.dealer_seed;
    const uint64_t cid = call_id(item_pair(m, it), step, it.layer, it.op, it.slot);
    if (m->d.mask_reuse && it.kind == IT_MATRIX && (it.op == OP_GRADW || it.op == OP_GRADIN))
        return deal_reuse_item(m, it, step, s);
    switch (it.kind) {
    case IT_MATRIX:
    case IT_CONV_FWD:
    case IT_CONV_GW:
        PSML_TRY(deal_prg(m, it, cid, s));
        return deal_gemm(m, it, s);
    case IT_HAD: {
        ProfScope prof(PROF_DEALER, s, (double)sizeof(T) * 6 * it.n);
        void *U[2] = {it.U.p[0], it.U.p[1]}, *V[2] = {it.V.p[0], it.V.p[1]}, *Z[2] = {it.Z.p[0], it.Z.p[1]};
        return hadamard_triplet_launch<T>(m->seeds, cid, it.n, U, V, Z, s, m->step_dev);
    }
    case IT_MSB: {
        ProfScope prof(PROF_DEALER, s, (double)sizeof(T) * 2 * it.mat.n);
        void *mt[2] = {it.mat.p[0], it.mat.p[1]};
        return msb_dealer_launch<T>(m->seeds, cid, it.n, mt, s, m->step_dev);
    }
    case IT_FSS: {
        ProfScope prof(PROF_DEALER, s, 2.0 * FSS_BITS * (double)it.n);
        if (!strong_rows(m, it)) return fss_dealer_launch(m->seeds, cid, it.n, it.mat.p[0], it.mat.p[1], s, m->step_dev);
        const int parts = item_parts(it);
        const int64_t per = it.n / parts;
        for (int h = 0; h < parts; ++h)   // local [h per, (h + 1) per) <- global part h, this pair's rows
            PSML_TRY(fss_dealer_launch(m->seeds, cid, it.n, it.mat.p[0], it.mat.p[1], s, m->step_dev, h * per,
                                       (h + 1) * per, strong_elem0(m, per, h) - h * per));
        return PSML_OK;
    }
    }
    return PSML_OK;
}

// Work lists of the fused dealer for items[pool] (step field of the call ids filled in on device).
static psml_status build_plan(psml_model_s *m, int pool, bool infer_only) {
    DealPlan &P = m->plan[pool][infer_only ? 1 : 0];
    // cluster split of the dealer's grouped Z = U V launch: 4 (measured vs 2 and 8: 919K vs
    // 895K / 897K samples/s); 32 x 32 tiles (64 x 64 tiles measured 720K: their CTAs crowd out the
    // online chain)
    P.gemm_ks = 4;
    P.gemm_big = false;
    const int gBM = P.gemm_big ? ClDealer::BM : ClDefault::BM, gBN = P.gemm_big ? ClDealer::BN : ClDefault::BN;
    const int gBK = P.gemm_big ? ClDealer::BK : ClDefault::BK;
    std::vector<PrgJob> pjm, pjr;   // matrix-triplet streams, then the rest
    std::vector<ClJob<DealerOps<T>>> gj;
    // one job: n elements of every stream in `tags`, stream element e0 = boff * 8 first
    auto job = [&](int kind, std::initializer_list<uint32_t> tags, uint64_t cid, int64_t n,
                   std::initializer_list<T *> outs, int64_t boff) {
        if (n <= 0) return;
        PrgJob j{};
        j.kind = kind;
        j.mask = ~(uint64_t)0;
        int i = 0;
        for (uint32_t t : tags) j.tag[i++] = t;
        i = 0;
        for (T *o : outs) j.out[i++] = o;
        j.cid = cid; j.n = n; j.boff = boff;
        P.chacha_blocks += (double)((n + 7) / 8) * (double)tags.size();
        (kind == PJ_PAIR || kind == PJ_SINGLE ? pjm : pjr).push_back(j);
    };
    auto &items = m->items[pool];
    for (size_t k = 0; k < items.size(); ++k) {
        DealItem &it = items[k];
        if (infer_only && !it.fwd) continue;
        const uint64_t cid = call_id(item_pair(m, it), 0, it.layer, it.op, it.slot);
        // strong scaling (R28): this pair's rows of the global streams; U and Z row-sliced, V global
        const bool sr = strong_rows(m, it);
        const int parts = sr ? item_parts(it) : 1;
        const int64_t kp = m->d.pair_id;
        switch (it.kind) {
        case IT_MATRIX:
        case IT_CONV_FWD:
        case IT_CONV_GW: {
            job(PJ_PAIR, {TAG_U0, TAG_U1}, cid, it.U.n, {it.U.p[0], it.U.p[1]}, sr ? kp * it.U.n / 8 : 0);
            job(PJ_PAIR, {TAG_V0, TAG_V1}, cid, it.V.n, {it.V.p[0], it.V.p[1]}, 0);
            job(PJ_SINGLE, {TAG_Z0}, cid, it.Z.n, {it.Z.p[0]}, sr ? kp * it.Z.n / 8 : 0);
            if (it.kind == IT_MATRIX && !m->ctx->use_tc(it.M, it.K, it.N) && it.M * it.N > 0) {
                ClJob<DealerOps<T>> g{};
                g.ops.U0 = it.U.p[0]; g.ops.U1 = it.U.p[1]; g.ops.V0 = it.V.p[0]; g.ops.V1 = it.V.p[1];
                g.ops.Z0 = it.Z.p[0]; g.ops.Z1 = it.Z.p[1];
                g.ops.M = it.M; g.ops.N = it.N; g.ops.Kext = it.K;
                g.tiles_n = (int)((it.N + gBN - 1) / gBN);
                g.tile_begin = P.gemm_tiles;
                g.k_per_split = ((it.K + P.gemm_ks - 1) / P.gemm_ks + gBK - 1) / gBK * gBK;
                P.gemm_tiles += ((it.M + gBM - 1) / gBM) * g.tiles_n;
                gj.push_back(g);
            } else {
                P.rest.push_back((int)k);
            }
            break;
        }
        case IT_HAD: {
            const int64_t per = it.n / parts;
            for (int h = 0; h < parts; ++h) {
                const int64_t q = h * per;   // local part h <- global part h, this pair's rows
                job(PJ_HAD, {TAG_U0, TAG_U1, TAG_V0, TAG_V1, TAG_Z0}, cid, per,
                    {it.U.p[0] + q, it.U.p[1] + q, it.V.p[0] + q, it.V.p[1] + q, it.Z.p[0] + q, it.Z.p[1] + q},
                    sr ? strong_elem0(m, per, h) / 8 : 0);
            }
            break;
        }
        case IT_MSB: {   // the reduced prefix's 3 AND groups + the daBit (R27); planes of n
            T *m0 = it.mat.p[0], *m1 = it.mat.p[1];
            const int64_t n = it.n, per = n / parts;
            for (int h = 0; h < parts; ++h) {
                const int64_t q = h * per, bo = sr ? strong_elem0(m, per, h) / 8 : 0;
                for (int g = 0; g < 3; ++g) {
                    const int64_t o = (int64_t)g * 3 * n + q;
                    job(PJ_AND, {tag4('a', '0', g), tag4('a', '1', g), tag4('b', '0', g), tag4('b', '1', g), tag4('c', '0', g)},
                        cid, per, {m0 + o, m1 + o, m0 + o + n, m1 + o + n, m0 + o + 2 * n, m1 + o + 2 * n}, bo);
                    pjr.back().mask = msb_group_mask(64, g);
                }
                const int64_t o = (int64_t)9 * n + q;
                job(PJ_DABIT, {TAG_R0, TAG_R1, TAG_RA}, cid, per, {m0 + o, m1 + o, m0 + o + n, m1 + o + n}, bo);
            }
            break;
        }
        case IT_FSS:
            P.fss.push_back((int)k);
            break;
        }
    }
    std::vector<PrgJob> pj(pjm);
    pj.insert(pj.end(), pjr.begin(), pjr.end());
    P.n_prg_mat = (int)pjm.size();
    for (size_t i = 0; i < pj.size(); ++i) {
        pj[i].blk_begin = P.prg_blocks;
        P.prg_blocks += (pj[i].n + 7) / 8;
        if ((int)i + 1 == P.n_prg_mat) P.prg_mat_blocks = P.prg_blocks;
    }
    P.n_prg = (int)pj.size();
    P.n_gemm = (int)gj.size();
    if (P.n_prg) {
        T *d = nullptr;
        PSML_TRY(dalloc(m, &d, (int64_t)((sizeof(PrgJob) * pj.size() + 7) / 8)));
        PSML_CUDA_TRY(cudaMemcpy(d, pj.data(), sizeof(PrgJob) * pj.size(), cudaMemcpyHostToDevice));
        P.prg = (PrgJob *)d;
    }
    if (P.n_gemm) {
        T *d = nullptr;
        const size_t bytes = sizeof(ClJob<DealerOps<T>>) * gj.size();
        PSML_TRY(dalloc(m, &d, (int64_t)((bytes + 7) / 8)));
        PSML_CUDA_TRY(cudaMemcpy(d, gj.data(), bytes, cudaMemcpyHostToDevice));
        P.gemm = (ClJob<DealerOps<T>> *)d;
    }
    return PSML_OK;
}

// second dealer branch inside a pipelined capture (psml_options.deal_split = 0: one branch)
static cudaStream_t deal_s2(psml_model_s *m) { return cur_opts().deal_split ? m->side2 : nullptr; }

// PRG jobs [j0, j1) (blocks [b0, b1)) of plan P on stream s
static psml_status deal_prg_launch(psml_model_s *m, const DealPlan &P, int j0, int j1, int64_t b0, int64_t b1,
                                   cudaStream_t s, bool second = false) {
    if (j1 <= j0 || b1 <= b0) return PSML_OK;
    // a bounded grid (grid-stride): the PRG work runs beside the online phase instead of
    // occupying every SM's register file ahead of it
    const int per_sm1 = 4;   // CTAs per SM, measured best of {1, 2, 4, full grid}
    const int per_sm2 = 2;   // second branch: best of {2, 3, 4}
    // (the CNN's dealer is most of its step: both of its branches keep the full budget -- 56.3K vs
    // 54.7K samples/s with the MLP's split)
    const int per_sm = (second && m->d.kind != PSML_CNN) ? per_sm2 : per_sm1;
    const int64_t full = (b1 - b0 + 127) / 128;
    // a dealer forked after the whole online chain (models without the fused step, e.g. the CNN)
    // overlaps nothing but the update: it takes the whole GPU
    const int64_t grid = (per_sm > 0 && !m->deal_alone) ? std::min<int64_t>(full, (int64_t)per_sm * m->ctx->sm_count)
                                                        : full;
    deal_prg_kernel<<<(unsigned)grid, 128, 0, s>>>(P.prg + j0, j1 - j0, b0, b1, m->seeds, m->step_dev);
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

// Dealer of one pool.  With a second stream s2 (the pipelined graph), the AND / daBit / Hadamard
// streams run on s2 while s runs the matrix-triplet streams and then Z = U V, so the products'
// material is ready early; s joins s2 before returning.
static psml_status deal_pool(psml_model_s *m, int pool, uint32_t step, bool infer_only, cudaStream_t s,
                             cudaStream_t s2 = nullptr) {
    if (m->d.strong_pairs > 1 && !fused_deal())
        return fail(PSML_ERR_UNSUPPORTED, "strong scaling: the row-sliced material needs the fused dealer");
    if (!fused_deal() || m->d.mask_reuse) {   // mask reuse: the backward triplets copy forward masks
        for (auto &it : m->items[pool]) {
            if (infer_only && !it.fwd) continue;
            PSML_TRY(deal_item(m, it, step, s));
        }
        return PSML_OK;
    }
    (void)step;   // the step field comes from m->step_dev (set by the caller / the graph)
    DealPlan &P = m->plan[pool][infer_only ? 1 : 0];
    const bool fork = s2 && P.n_prg_mat > 0 && P.n_prg > P.n_prg_mat;
    {
        ProfScope prof(PROF_DEALER, s, P.chacha_blocks);   // work = ChaCha20 blocks of the step
        if (fork) {
            // the matrix-triplet streams (needed by the Z = U V launch that follows them) are
            // created first so they are scheduled first; the second branch forks from before them
            PSML_CUDA_TRY(cudaEventRecord(m->ev_d2, s));
            PSML_TRY(deal_prg_launch(m, P, 0, P.n_prg_mat, 0, P.prg_mat_blocks, s));
            PSML_CUDA_TRY(cudaStreamWaitEvent(s2, m->ev_d2, 0));
            PSML_TRY(deal_prg_launch(m, P, P.n_prg_mat, P.n_prg, P.prg_mat_blocks, P.prg_blocks, s2, true));
            PSML_CUDA_TRY(cudaEventRecord(m->ev_d2j, s2));
        } else {
            PSML_TRY(deal_prg_launch(m, P, 0, P.n_prg, 0, P.prg_blocks, s));
        }
        if (P.n_gemm) {
            cudaLaunchConfig_t cfg = {};
            cfg.gridDim = dim3((unsigned)P.gemm_tiles, 1, (unsigned)P.gemm_ks);
            cfg.blockDim = dim3(P.gemm_big ? ClDealer::NT : ClDefault::NT);
            cfg.stream = s;
            cudaLaunchAttribute attr[1];
            attr[0].id = cudaLaunchAttributeClusterDimension;
            attr[0].val.clusterDim.x = 1; attr[0].val.clusterDim.y = 1; attr[0].val.clusterDim.z = (unsigned)P.gemm_ks;
            cfg.attrs = attr;
            cfg.numAttrs = 1;
            if (P.gemm_big)
                PSML_CUDA_TRY(cudaLaunchKernelEx(&cfg, ring_gemm_cl_grouped<T, DealerOps<T>, ClDealer>,
                                                 (const ClJob<DealerOps<T>> *)P.gemm, P.n_gemm, P.gemm_ks));
            else
                PSML_CUDA_TRY(cudaLaunchKernelEx(&cfg, ring_gemm_cl_grouped<T, DealerOps<T>>,
                                                 (const ClJob<DealerOps<T>> *)P.gemm, P.n_gemm, P.gemm_ks));
        }
    }
    for (int k : P.rest) PSML_TRY(deal_gemm(m, m->items[pool][k], s));
    for (int k : P.fss) PSML_TRY(deal_item(m, m->items[pool][k], 0, s));   // step from m->step_dev
    if (fork) PSML_CUDA_TRY(cudaStreamWaitEvent(s, m->ev_d2j, 0));
    return PSML_OK;
}

// ------------------------------------------------------------------------------------------------
// online pieces
// ------------------------------------------------------------------------------------------------
static psml_status mm(psml_model_s *m, const T *const A[2], const T *const Bm[2], int layer, int op, int flags,
                      int trunc, T *const C[2], cudaStream_t s) {
    DealItem *it = find_item(m, layer, op, 0);
    if (!it) return fail(PSML_ERR_STATE, "missing triplet");
    if (m->ctx->use_tc(it->M, 2 * it->K, it->N))
        return tc_beaver_matmul_ws<T>(A, Bm, it->U.cp(), it->V.cp(), it->Z.cp(), it->M, it->K, it->N, flags, trunc, C,
                                      m->ws, sizeof(T) * (size_t)m->ws_words, m->ctx->sm_count, s);
    if (fused_open())   // co-resident: mask round fused into the GEMM's operand loads
        return beaver_matmul_fused<T>(A, Bm, it->U.cp(), it->V.cp(), it->Z.cp(), it->M, it->K, it->N, flags, trunc, C,
                                      m->ws, m->ws_words, s, m->ctx->sm_count);
    return beaver_matmul<T>(A, Bm, it->U.cp(), it->V.cp(), it->Z.cp(), it->M, it->K, it->N, flags, trunc, C, m->ws,
                            m->ws_words, s, m->ctx->sm_count);
}

// FSS ReLU (R22) of n elements, both parties: DReLU from one opening, then the Beaver Hadamard.
// ws: 8 n words.
static psml_status relu_fss(const T *const x[2], int64_t n, const DealItem *mat, const DealItem *h, T *const y[2],
                            T *const dr[2], T *ws, cudaStream_t s) {
    T *d[2] = {dr ? dr[0] : ws + 2 * n, dr ? dr[1] : ws + 3 * n};
    PSML_TRY(fss_drelu_launch(CPair<T>{{x[0], x[1]}}, n, CPair<T>{{mat->mat.p[0], mat->mat.p[1]}}, Pair<T>{{d[0], d[1]}},
                              nullptr, ws, s));
    const T *dc[2] = {d[0], d[1]};
    return beaver_hadamard<T>(x, dc, h->U.cp(), h->V.cp(), h->Z.cp(), n, 0, y, ws + 4 * n, s);
}

static psml_status relu(psml_model_s *m, const T *const x[2], int layer, T *const y[2], T *const dr[2],
                        cudaStream_t s) {
    DealItem *mat = find_item(m, layer, OP_RELU_MSB, 0), *h = find_item(m, layer, OP_HADAMARD, 0);
    if (!mat || !h) return fail(PSML_ERR_STATE, "missing ReLU material");
    if (mat->kind == IT_FSS) return relu_fss(x, mat->n, mat, h, y, dr, m->ws, s);
    return msb_chain<T>(x, mat->n, mat->mat.cp(), 0, 0, 1, nullptr, nullptr, dr, h->U.cp(), h->V.cp(), h->Z.cp(), y,
                        nullptr, nullptr, m->ws, s);
}

static psml_status eq9(psml_model_s *m, const T *const z[2], int layer, T *const y[2], const T *const Y[2],
                       T *const dlt[2], cudaStream_t s) {
    DealItem *mat = find_item(m, layer, OP_EQ9_MSB, 0), *h = find_item(m, layer, OP_HADAMARD, 2);
    if (!mat || !h) return fail(PSML_ERR_STATE, "missing Eq. 9 material");
    const T half = (T)1 << (m->ctx->ring.frac_bits - 1);
    if (mat->kind == IT_FSS) {   // Eq. 9 = ReLU(z + 1/2) - ReLU(z - 1/2) with the FSS ReLU (R22)
        const int64_t n2 = mat->n, n = n2 / 2;
        T *xin[2] = {m->ws + 8 * n2, m->ws + 9 * n2}, *r[2] = {m->ws + 10 * n2, m->ws + 11 * n2};
        eq9_prep_kernel<<<ew_grid(n), EW_THREADS, 0, s>>>(CPair<T>{{z[0], z[1]}}, n, half, Pair<T>{{xin[0], xin[1]}}, -1);
        PSML_LAUNCH_CHECK();
        const T *xc[2] = {xin[0], xin[1]};
        PSML_TRY(relu_fss(xc, n2, mat, h, r, nullptr, m->ws, s));
        eq9_combine_kernel<<<ew_grid(n), EW_THREADS, 0, s>>>(CPair<T>{{r[0], r[1]}}, n, Pair<T>{{y[0], y[1]}},
                                                              CPair<T>{{Y ? Y[0] : nullptr, Y ? Y[1] : nullptr}},
                                                              Pair<T>{{dlt ? dlt[0] : nullptr, dlt ? dlt[1] : nullptr}}, -1);
        PSML_LAUNCH_CHECK();
        return PSML_OK;
    }
    return msb_chain<T>(z, mat->n, mat->mat.cp(), 1, half, 2, nullptr, nullptr, nullptr, h->U.cp(), h->V.cp(),
                        h->Z.cp(), y, Y, dlt, m->ws, s);
}

static psml_status had(psml_model_s *m, const T *const a[2], const T *const b[2], int layer, int slot, T *const c[2],
                       cudaStream_t s) {
    DealItem *h = find_item(m, layer, OP_HADAMARD, slot);
    if (!h) return fail(PSML_ERR_STATE, "missing Hadamard triplet");
    return beaver_hadamard<T>(a, b, h->U.cp(), h->V.cp(), h->Z.cp(), h->n, 0, c, m->ws, s);
}

static psml_status sub(const T *const a[2], const T *const b[2], int64_t n, T *const c[2], cudaStream_t s) {
    sub_pair_kernel<T><<<ew_grid(n), EW_THREADS, 0, s>>>(CPair<T>{{a[0], a[1]}}, CPair<T>{{b[0], b[1]}}, n,
                                                          Pair<T>{{c[0], c[1]}});
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

static psml_status conv(psml_model_s *m, const T *const X[2], const T *const Bm[2], int transposed, int trunc,
                        T *const C[2], cudaStream_t s) {
    DealItem *it = find_item(m, 0, transposed ? OP_GRADW : OP_FWD, 0);
    if (!it) return fail(PSML_ERR_STATE, "missing conv triplet");
    return conv_beaver<T>(X, Bm, it->U.cp(), it->V.cp(), it->Z.cp(), m->B, m->g, transposed, it->N, trunc, C, m->ws,
                          m->ws_words, s, m->ctx->sm_count);
}

static T *const *gradp(psml_model_s *m, int layer, T *tmp[2]) {
    tmp[0] = m->grad_base + m->grad_off[layer];
    tmp[1] = m->grad_base + m->grad_words + m->grad_off[layer];
    return tmp;
}

using T_ = T;
// RNN input of step t: A[b, 0:D] = X[b, t D : (t + 1) D], A[b, D:D+H] = h_prev[b, :] (0 at t = 0)
static __global__ void rnn_concat_kernel(CPair<T> X, CPair<T> hprev, int64_t B, int64_t D, int64_t H, int64_t xw, int t,
                                         Pair<T> A) {
    const int64_t K = D + H, n = B * K;
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n; e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t b = e / K, k = e % K;
#pragma unroll
        for (int p = 0; p < 2; ++p)
            A.p[p][e] = k < D ? X.p[p][b * xw + (int64_t)t * D + k] : (hprev.p[p] ? hprev.p[p][b * H + (k - D)] : (T)0);
    }
}
static __global__ void add_pair_kernel(CPair<T> a, CPair<T> b, int64_t n, Pair<T> c) {
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n; e += (int64_t)gridDim.x * blockDim.x)
#pragma unroll
        for (int p = 0; p < 2; ++p) c.p[p][e] = a.p[p][e] + b.p[p][e];
}

// out_p = (neg ? -in_p : in_p) + [p == 0] c   (public constants are added by party 0)
static __global__ void affine_pair_kernel(CPair<T> in, int64_t n, T c, int neg, Pair<T> out) {
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n; e += (int64_t)gridDim.x * blockDim.x)
#pragma unroll
        for (int p = 0; p < 2; ++p) {
            const T v = neg ? (T)0 - in.p[p][e] : in.p[p][e];
            out.p[p][e] = p == 0 ? v + c : v;
        }
}

// Linear SVM (R24): m = trunc(y (.) z, F); ind = [m - 1 < 0]; delta = -(y (.) ind).
static psml_status svm_delta(psml_model_s *m, const T *const z[2], const T *const Y[2], cudaStream_t s) {
    const int F = m->ctx->ring.frac_bits;
    const int64_t n = m->B;
    DealItem *h3 = find_item(m, 0, OP_HADAMARD, 3), *h4 = find_item(m, 0, OP_HADAMARD, 4);
    DealItem *cmp = find_item(m, 0, OP_RELU_MSB, 0);
    if (!h3 || !h4 || !cmp) return fail(PSML_ERR_STATE, "missing SVM material");
    T *mg[2] = {m->tmp.p[0], m->tmp.p[1]};                 // margin, then m - 1
    T *ind[2] = {m->tmp.p[0] + n, m->tmp.p[1] + n};
    T *c[2] = {m->tmp.p[0] + 2 * n, m->tmp.p[1] + 2 * n};
    T *ws = m->ws;
    PSML_TRY(beaver_hadamard<T>(Y, z, h3->U.cp(), h3->V.cp(), h3->Z.cp(), n, F, mg, ws, s));
    affine_pair_kernel<<<ew_grid(n), EW_THREADS, 0, s>>>(CPair<T>{{mg[0], mg[1]}}, n, (T)0 - ((T)1 << F), 0,
                                                         Pair<T>{{mg[0], mg[1]}});
    PSML_LAUNCH_CHECK();
    const T *t[2] = {mg[0], mg[1]};
    if (cmp->kind == IT_FSS) {   // [t < 0] = 1 - DReLU(t)
        PSML_TRY(fss_drelu_launch(CPair<T>{{t[0], t[1]}}, n, CPair<T>{{cmp->mat.p[0], cmp->mat.p[1]}},
                                  Pair<T>{{ind[0], ind[1]}}, nullptr, ws, s));
        affine_pair_kernel<<<ew_grid(n), EW_THREADS, 0, s>>>(CPair<T>{{ind[0], ind[1]}}, n, (T)1, 1,
                                                             Pair<T>{{ind[0], ind[1]}});
        PSML_LAUNCH_CHECK();
    } else {                     // the A2B chain's arithmetic MSB shares
        PSML_TRY(msb_chain<T>(t, n, cmp->mat.cp(), 0, 0, 0, ind, nullptr, nullptr, nullptr, nullptr, nullptr,
                              nullptr, nullptr, nullptr, ws, s));
    }
    const T *ic[2] = {ind[0], ind[1]};
    PSML_TRY(beaver_hadamard<T>(Y, ic, h4->U.cp(), h4->V.cp(), h4->Z.cp(), n, 0, c, ws, s));
    affine_pair_kernel<<<ew_grid(n), EW_THREADS, 0, s>>>(CPair<T>{{c[0], c[1]}}, n, (T)0, 1,
                                                         Pair<T>{{m->delta.p[0], m->delta.p[1]}});
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

// forward pass; if Y != nullptr also leaves delta = yhat - Y in m->delta
static psml_status forward(psml_model_s *m, const T *const X[2], const T *const Y[2], T *const out[2],
                           cudaStream_t s) {
    const int F = m->ctx->ring.frac_bits;
    m->act[0].p[0] = (T *)X[0];
    m->act[0].p[1] = (T *)X[1];
    T *yo[2] = {out ? out[0] : m->yhat.p[0], out ? out[1] : m->yhat.p[1]};
    if (m->d.kind == PSML_RNN) {
        const int T = m->rnn_T;
        const int64_t D = m->rnn_D, H = m->dims[1], K1 = m->rows[0], B = m->B;
        for (int t = 1; t <= T; ++t) {
            T_ *At[2] = {m->rnnA.p[0] + (t - 1) * B * K1, m->rnnA.p[1] + (t - 1) * B * K1};
            const T_ *hp[2] = {t > 1 ? m->rnnH.p[0] + (t - 2) * B * H : nullptr, t > 1 ? m->rnnH.p[1] + (t - 2) * B * H : nullptr};
            rnn_concat_kernel<<<ew_grid(B * K1), EW_THREADS, 0, s>>>(CPair<T_>{{X[0], X[1]}}, CPair<T_>{{hp[0], hp[1]}}, B, D,
                                                                    H, (int64_t)m->dims[0], t - 1, Pair<T_>{{At[0], At[1]}});
            PSML_LAUNCH_CHECK();
            const T_ *Ac[2] = {At[0], At[1]};
            PSML_TRY(mm(m, Ac, m->W[0].cp(), t, OP_FWD, 0, fw(m, 0), m->z[0].pp(), s));
            T_ *ht[2] = {m->rnnH.p[0] + (t - 1) * B * H, m->rnnH.p[1] + (t - 1) * B * H};
            T_ *dt[2] = {m->rnnD.p[0] + (t - 1) * B * H, m->rnnD.p[1] + (t - 1) * B * H};
            PSML_TRY(relu(m, m->z[0].cp(), t, ht, dt, s));
        }
        const T_ *hT[2] = {m->rnnH.p[0] + (T - 1) * B * H, m->rnnH.p[1] + (T - 1) * B * H};
        PSML_TRY(mm(m, hT, m->W[1].cp(), T + 1, OP_FWD, 0, fw(m, 1), m->z[1].pp(), s));
        return eq9(m, m->z[1].cp(), T + 1, yo, Y, Y ? m->delta.pp() : nullptr, s);
    }
    if (m->d.kind == PSML_SVM) {
        PSML_TRY(mm(m, m->act[0].cp(), m->W[0].cp(), 0, OP_FWD, 0, fw(m, 0), m->z[0].pp(), s));
        const int64_t n = m->B;
        for (int p = 0; p < 2; ++p)
            PSML_CUDA_TRY(cudaMemcpyAsync(yo[p], m->z[0].p[p], sizeof(T) * n, cudaMemcpyDeviceToDevice, s));
        return Y ? svm_delta(m, m->z[0].cp(), Y, s) : PSML_OK;
    }
    if (m->d.kind == PSML_CNN) {
        PSML_TRY(conv(m, X, m->W[0].cp(), 0, fw(m, 0), m->z[0].pp(), s));
        PSML_TRY(relu(m, m->z[0].cp(), 0, m->act[1].pp(), m->drelu[0].pp(), s));
        PSML_TRY(mm(m, m->act[1].cp(), m->W[1].cp(), 1, OP_FWD, 0, fw(m, 1), m->z[1].pp(), s));
        PSML_TRY(relu(m, m->z[1].cp(), 1, m->act[2].pp(), m->drelu[1].pp(), s));
        PSML_TRY(mm(m, m->act[2].cp(), m->W[2].cp(), 2, OP_FWD, 0, fw(m, 2), m->z[2].pp(), s));
        return eq9(m, m->z[2].cp(), 2, yo, Y, Y ? m->delta.pp() : nullptr, s);
    }
    const int nl = m->nl;
    for (int l = 0; l < nl; ++l) {
        PSML_TRY(mm(m, m->act[l].cp(), m->W[l].cp(), l, OP_FWD, 0, fw(m, l), m->z[l].pp(), s));
        if (l < nl - 1) {
            PSML_TRY(relu(m, m->z[l].cp(), l, m->act[l + 1].pp(), m->drelu[l].pp(), s));
        } else if (is_eq9_out(m)) {
            PSML_TRY(eq9(m, m->z[l].cp(), l, yo, Y, Y ? m->delta.pp() : nullptr, s));
        } else {
            const int64_t n = m->B * m->dims[nl];
            for (int p = 0; p < 2; ++p)
                PSML_CUDA_TRY(cudaMemcpyAsync(yo[p], m->z[l].p[p], sizeof(T) * n, cudaMemcpyDeviceToDevice, s));
            if (Y) PSML_TRY(sub(m->z[l].cp(), Y, n, m->delta.pp(), s));
        }
    }
    return PSML_OK;
}

static psml_status backward(psml_model_s *m, cudaStream_t s) {
    const int F = m->ctx->ring.frac_bits;
    T *g[2];
    if (m->d.kind == PSML_SVM)
        return mm(m, m->act[0].cp(), m->delta.cp(), 0, OP_GRADW, PSML_TRANS_A, 0, gradp(m, 0, g), s);
    if (m->d.kind == PSML_RNN) {   // backpropagation through time (R25)
        const int T = m->rnn_T;
        const int64_t D = m->rnn_D, H = m->dims[1], K1 = m->rows[0], B = m->B;
        const T_ *hT[2] = {m->rnnH.p[0] + (T - 1) * B * H, m->rnnH.p[1] + (T - 1) * B * H};
        PSML_TRY(mm(m, hT, m->delta.cp(), T + 1, OP_GRADW, PSML_TRANS_A, 0, gradp(m, 1, g), s));
        PSML_TRY(mm(m, m->delta.cp(), m->W[1].cp(), T + 1, OP_GRADIN, PSML_TRANS_B, fw(m, 1), m->tmp.pp(), s));
        const T_ *dT[2] = {m->rnnD.p[0] + (T - 1) * B * H, m->rnnD.p[1] + (T - 1) * B * H};
        PSML_TRY(had(m, m->tmp.cp(), dT, T, 1, m->delta.pp(), s));
        T_ *g0[2];
        gradp(m, 0, g0);
        const T_ *Wh[2] = {m->W[0].p[0] + D * H, m->W[0].p[1] + D * H};   // W_h = rows D.. of W_1
        for (int t = T; t >= 1; --t) {
            const T_ *At[2] = {m->rnnA.p[0] + (t - 1) * B * K1, m->rnnA.p[1] + (t - 1) * B * K1};
            PSML_TRY(mm(m, At, m->delta.cp(), t, OP_GRADW, PSML_TRANS_A, 0, t == T ? g0 : m->rnnG.pp(), s));
            if (t < T) {   // gW_1 += A_t^T delta_t  (ring addition of untruncated shares)
                add_pair_kernel<<<ew_grid(K1 * H), EW_THREADS, 0, s>>>(CPair<T_>{{g0[0], g0[1]}},
                                                                      CPair<T_>{{m->rnnG.p[0], m->rnnG.p[1]}},
                                                                      K1 * H, Pair<T_>{{g0[0], g0[1]}});
                PSML_LAUNCH_CHECK();
            }
            if (t > 1) {
                PSML_TRY(mm(m, m->delta.cp(), Wh, t, OP_GRADIN, PSML_TRANS_B, fw(m, 0), m->tmp.pp(), s));
                const T_ *dp[2] = {m->rnnD.p[0] + (t - 2) * B * H, m->rnnD.p[1] + (t - 2) * B * H};
                PSML_TRY(had(m, m->tmp.cp(), dp, t - 1, 1, m->delta.pp(), s));
            }
        }
        return PSML_OK;
    }
    if (m->d.kind == PSML_CNN) {
        // layer 2 (FC 64 -> 10)
        PSML_TRY(mm(m, m->act[2].cp(), m->delta.cp(), 2, OP_GRADW, PSML_TRANS_A, 0, gradp(m, 2, g), s));
        PSML_TRY(mm(m, m->delta.cp(), m->W[2].cp(), 2, OP_GRADIN, PSML_TRANS_B, fw(m, 2), m->tmp.pp(), s));
        PSML_TRY(had(m, m->tmp.cp(), m->drelu[1].cp(), 1, 1, m->delta.pp(), s));
        // layer 1 (FC 12544 -> 64)
        PSML_TRY(mm(m, m->act[1].cp(), m->delta.cp(), 1, OP_GRADW, PSML_TRANS_A, 0, gradp(m, 1, g), s));
        PSML_TRY(mm(m, m->delta.cp(), m->W[1].cp(), 1, OP_GRADIN, PSML_TRANS_B, fw(m, 1), m->tmp.pp(), s));
        PSML_TRY(had(m, m->tmp.cp(), m->drelu[0].cp(), 0, 1, m->delta.pp(), s));
        // conv weight gradient: im2col(X)^T . delta   (delta viewed as (B*OH*OW) x Cout)
        return conv(m, m->act[0].cp(), m->delta.cp(), 1, 0, gradp(m, 0, g), s);
    }
    const int nl = m->nl;
    for (int l = nl - 1; l >= 0; --l) {
        PSML_TRY(mm(m, m->act[l].cp(), m->delta.cp(), l, OP_GRADW, PSML_TRANS_A, 0, gradp(m, l, g), s));
        if (l > 0) {
            PSML_TRY(mm(m, m->delta.cp(), m->W[l].cp(), l, OP_GRADIN, PSML_TRANS_B, fw(m, l), m->tmp.pp(), s));
            PSML_TRY(had(m, m->tmp.cp(), m->drelu[l - 1].cp(), l - 1, 1, m->delta.pp(), s));
        }
    }
    return PSML_OK;
}

// ------------------------------------------------------------------------------------------------
// fused co-resident training step (fused.cuh): MLP / linear / logistic regression
// ------------------------------------------------------------------------------------------------
static int item_index(const psml_model_s *m, int layer, int op, int slot) {
    for (size_t k = 0; k < m->items[0].size(); ++k) {
        const DealItem &it = m->items[0][k];
        if (it.layer == layer && it.op == op && it.slot == slot) return (int)k;
    }
    return -1;
}

static bool fused_eligible(const psml_model_s *m) {
    if (m->d.kind == PSML_CNN || m->d.kind == PSML_SVM || m->d.kind == PSML_RNN || m->nl > UPD_MAX_LAYERS ||
        (int)m->ob.size() != (int)m->items[0].size())
        return false;
    for (int l = 0; l < m->nl; ++l)
        if (fw(m, l) != m->ctx->ring.frac_bits) return false;   // the fused step truncates by F
    if (m->d.compare != 0) return false;                         // the fused step runs the A2B chain
    if (m->d.mask_reuse) return false;                           // ... and fresh backward masks
    return fuse_enabled() && chain_mode() == 0;
}

static bool fused_shapes_ok(const psml_model_s *m) {
    if (m->d.kind == PSML_CNN || m->nl > UPD_MAX_LAYERS) return false;
    for (auto &it : m->items[0])
        if (it.kind == IT_MATRIX && m->ctx->use_tc(it.M, 2 * it.K, it.N)) return false;
    return true;
}

static psml_status alloc_open_bufs(psml_model_s *m) {
    m->ob.assign(m->items[0].size(), OpenBuf{});
    for (size_t k = 0; k < m->items[0].size(); ++k) {
        const DealItem &it = m->items[0][k];
        if (it.kind != IT_MATRIX) continue;
        PSML_TRY(dalloc(m, &m->ob[k].E, it.M * it.K));
        PSML_TRY(dalloc(m, &m->ob[k].X1, it.M * it.K));
        PSML_TRY(dalloc(m, &m->ob[k].F, it.K * it.N));
    }
    return PSML_OK;
}

// Pipelined capture: the next step's dealer branch forks from the online chain after its
// `deal_after`-th stage (0 = at the start of the step), so the dealer's persistent PRG CTAs do not
// hold the SMs the first products need.
static psml_status deal_fork_point(psml_model_s *m, cudaStream_t s, bool force = false) {
    if (m->deal_pending_pool < 0) return PSML_OK;
    if (!force && ++m->deal_stage < m->deal_after) return PSML_OK;
    const int pool = m->deal_pending_pool;
    m->deal_pending_pool = -1;
    // ev_late = the fork edge: the completion of the online chain so far, or (deal_on_launch) the
    // launch completion of the product just launched -- all its CTAs resident, so its SMs are
    // taken before the dealer's grids arrive
    if (!m->fork_event_armed) PSML_CUDA_TRY(cudaEventRecord(m->ev_late, s));
    m->fork_event_armed = false;
    PSML_CUDA_TRY(cudaStreamWaitEvent(m->side, m->ev_late, 0));
    m->deal_alone = force;
    const psml_status st = deal_pool(m, pool, 0, false, m->side, deal_s2(m));
    m->deal_alone = false;
    PSML_TRY(st);
    advance_word_kernel<<<1, 1, 0, m->side>>>(m->step_dev);   // every reader of the word is done
    PSML_LAUNCH_CHECK();
    PSML_CUDA_TRY(cudaEventRecord(m->ev_join, m->side));
    return PSML_OK;
}


static bool gradw_branch() { return cur_opts().gradw_branch != 0; }

// both parties' shares [a | b] (n words each) to out: the client's read-back of the predictions
template <typename U>
__global__ void copy_pair_kernel(const U *__restrict__ a, const U *__restrict__ b, int64_t n, U *__restrict__ out) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < 2 * n; i += (int64_t)gridDim.x * blockDim.x)
        out[i] = i < n ? a[i] : b[i - n];
}
constexpr int OUT_GRID = 8;   // grid of the read-back node (2 B d_L words: a few KB)

static psml_status fused_forward_backward(psml_model_s *m, const T *const X[2], const T *const Y[2], cudaStream_t s) {
    const int F = m->ctx->ring.frac_bits;
    const int nl = m->nl;
    const int64_t B = m->B;
    auto &items = m->items[m->pool];
    auto idx = [&](int l, int op, int slot = 0) { return item_index(m, l, op, slot); };
    for (int l = 0; l < nl; ++l)
        if (idx(l, OP_FWD) < 0 || idx(l, OP_GRADW) < 0 || (l > 0 && idx(l, OP_GRADIN) < 0))
            return fail(PSML_ERR_STATE, "fused step: missing triplet");
    m->act[0].p[0] = (T *)X[0];
    m->act[0].p[1] = (T *)X[1];
    auto seg = [&](int l, int op, T *C0, T *C1, int trunc) {
        const int k = idx(l, op);
        const DealItem &it = items[k];
        const OpenBuf &o = m->ob[k];
        SegArgs<T> a{};
        a.X[0] = it.U.p[0]; a.X[1] = o.X1; a.E = o.E; a.F = o.F;
        for (int p = 0; p < 2; ++p) { a.V[p] = it.V.p[p]; a.Z[p] = it.Z.p[p]; a.party[p] = p; }
        a.C[0] = C0; a.C[1] = C1;
        a.M = it.M; a.N = it.N; a.K = it.K; a.trunc = trunc; a.nparty = 2;
        return a;
    };
    // A side of product (l, op): mask U, outputs E, X_1;  B side: mask V, output F
    auto emitA = [&](int l, int op, int64_t rows, int64_t cols, int trans) {
        const int k = idx(l, op);
        Emit<T> e{};
        e.M[0] = items[k].U.p[0]; e.M[1] = items[k].U.p[1];
        e.E = m->ob[k].E; e.X1 = m->ob[k].X1; e.rows = rows; e.cols = cols; e.trans = trans;
        return e;
    };
    auto emitB = [&](int l, int op, int64_t rows, int64_t cols) {
        const int k = idx(l, op);
        Emit<T> e{};
        e.M[0] = items[k].V.p[0]; e.M[1] = items[k].V.p[1];
        e.E = m->ob[k].F; e.X1 = nullptr; e.rows = rows; e.cols = cols; e.trans = 0;
        return e;
    };
    // 1. step-start opens: the input batch and every weight matrix
    {
        OpenList<T> L{};
        int n = 0;
        int64_t tiles = 0;
        auto add = [&](const T *s0, const T *s1, const T *m0, const T *m1, T *open, T *x, int64_t rows, int64_t cols,
                       int trans) {
            OpenJob<T> &j = L.j[n];
            j.src[0] = s0; j.src[1] = s1; j.mask[0] = m0; j.mask[1] = m1;
            j.open = open; j.x = x; j.xmask = x ? m1 : nullptr; j.scale = 1;
            j.rows = rows; j.cols = cols; j.trans = trans;
            L.tile_begin[n] = tiles;
            tiles += ((rows + 31) / 32) * ((cols + 31) / 32);
            ++n;
        };
        {
            const int k = idx(0, OP_FWD);
            add(X[0], X[1], items[k].U.p[0], items[k].U.p[1], m->ob[k].E, m->ob[k].X1, B, m->dims[0], 0);
            const int g = idx(0, OP_GRADW);   // op(A) = X^T (d_0 x B), X stored B x d_0
            add(X[0], X[1], items[g].U.p[0], items[g].U.p[1], m->ob[g].E, m->ob[g].X1, m->dims[0], B, 1);
        }
        for (int l = 0; l < nl; ++l) {
            const int k = idx(l, OP_FWD);
            add(m->W[l].p[0], m->W[l].p[1], items[k].V.p[0], items[k].V.p[1], m->ob[k].F, nullptr, m->dims[l],
                m->dims[l + 1], 0);
            if (l > 0) {   // op(B) = W_l^T (d_{l+1} x d_l), W_l stored d_l x d_{l+1}
                const int g = idx(l, OP_GRADIN);
                add(m->W[l].p[0], m->W[l].p[1], items[g].V.p[0], items[g].V.p[1], m->ob[g].F, nullptr,
                    m->dims[l + 1], m->dims[l], 1);
            }
        }
        L.n = n;
        L.tile_begin[n] = tiles;
        ProfScope prof(PROF_MASK, s, 0.0);
        PSML_CUDA_TRY(launch_pdl(open_list_kernel<T>, dim3((unsigned)tiles), dim3(32, 8), s, L));
        PSML_LAUNCH_CHECK();
        PSML_TRY(deal_fork_point(m, s));
    }
    // 2. forward
    T *yo[2] = {m->yhat.p[0], m->yhat.p[1]};
    for (int l = 0; l < nl; ++l) {
        SegArgs<T> a = seg(l, OP_FWD, m->z[l].p[0], m->z[l].p[1], F);
        const bool arm = l == 0 && m->deal_on_launch && m->deal_pending_pool >= 0;
        if (arm) arm_launch_event(m->ev_late);
        PSML_TRY(launch_seg_group<T>(&a, 1, s, m->ctx->sm_count));
        if (arm) {
            m->fork_event_armed = take_launch_event() == nullptr;   // consumed by a tcgen05 launch
            if (m->fork_event_armed) m->deal_stage = m->deal_after - 1;   // fork right here
        }
        PSML_TRY(deal_fork_point(m, s));
        const int64_t w = m->dims[l + 1];
        if (l < nl - 1) {
            Emits<T> em{};
            em.e[0] = emitA(l + 1, OP_FWD, B, w, 0);
            em.e[1] = emitA(l + 1, OP_GRADW, B, w, 1);
            em.n = 2;
            DealItem *mat = find_item(m, l, OP_RELU_MSB, 0), *h = find_item(m, l, OP_HADAMARD, 0);
            if (!mat || !h) return fail(PSML_ERR_STATE, "missing ReLU material");
            PSML_TRY(msb_chain<T>(m->z[l].cp(), mat->n, mat->mat.cp(), 0, 0, 1, nullptr, nullptr, m->drelu[l].pp(),
                                  h->U.cp(), h->V.cp(), h->Z.cp(), m->act[l + 1].pp(), nullptr, nullptr, m->ws, s,
                                  &em));
            PSML_TRY(deal_fork_point(m, s));
        } else {
            Emits<T> em{};
            em.e[0] = emitB(l, OP_GRADW, B, w);
            em.n = 1;
            if (l > 0) { em.e[1] = emitA(l, OP_GRADIN, B, w, 0); em.n = 2; }
            if (is_eq9_out(m)) {
                DealItem *mat = find_item(m, l, OP_EQ9_MSB, 0), *h = find_item(m, l, OP_HADAMARD, 2);
                if (!mat || !h) return fail(PSML_ERR_STATE, "missing Eq. 9 material");
                const T half = (T)1 << (F - 1);
                PSML_TRY(msb_chain<T>(m->z[l].cp(), mat->n, mat->mat.cp(), 1, half, 2, nullptr, nullptr, nullptr,
                                      h->U.cp(), h->V.cp(), h->Z.cp(), yo, Y, m->delta.pp(), m->ws, s, &em));
            } else {
                DeltaFused<T> d{};
                for (int p = 0; p < 2; ++p) {
                    d.z[p] = m->z[l].p[p]; d.Y[p] = Y[p]; d.yhat[p] = yo[p]; d.delta[p] = m->delta.p[p];
                }
                d.n = B * w;
                d.em = em;
                PSML_CUDA_TRY(launch_pdl(delta_fused_kernel<T>, dim3(ew_grid(d.n)), dim3(EW_THREADS), s, d));
                PSML_LAUNCH_CHECK();
            }
        }
    }
    if (m->cap_out) {   // the read-back branch (a no-op until psml_model_step_host sets it)
        PSML_CUDA_TRY(cudaEventRecord(m->ev_y, s));
        PSML_CUDA_TRY(cudaStreamWaitEvent(m->d2h, m->ev_y, 0));
        copy_pair_kernel<T><<<OUT_GRID, 256, 0, m->d2h>>>(yo[0], yo[1], 0, nullptr);
        PSML_LAUNCH_CHECK();
        PSML_CUDA_TRY(cudaEventRecord(m->ev_yj, m->d2h));
    }
    // 3. backward: gradW_l and gradin_l in one launch, then the backprop Hadamard opens delta_{l-1}
    //    With PSML_GRADW_BRANCH (default on), gradW_l for l > 0 runs on a second stream as soon as
    //    delta_l is open, beside the chain gradin_l -> Hadamard -> ... that carries the backward
    //    dependency (the paper's inter-layer pipeline, Fig. 6, as stream overlap);
    //    the branch joins before the update.
    const bool branch = gradw_branch() && nl > 1;
    T *g[2];
    for (int l = nl - 1; l >= 0; --l) {
        gradp(m, l, g);
        SegArgs<T> jobs[2];
        jobs[0] = seg(l, OP_GRADW, g[0], g[1], 0);
        if (l > 0) jobs[1] = seg(l, OP_GRADIN, m->tmp.p[0], m->tmp.p[1], F);
        if (branch && l > 0) {
            PSML_CUDA_TRY(cudaEventRecord(m->ev_gw, s));
            PSML_CUDA_TRY(cudaStreamWaitEvent(m->gw, m->ev_gw, 0));
            PSML_TRY(launch_seg_group<T>(&jobs[0], 1, m->gw, m->ctx->sm_count));
            PSML_TRY(launch_seg_group<T>(&jobs[1], 1, s, m->ctx->sm_count));
        } else {
            PSML_TRY(launch_seg_group<T>(jobs, l > 0 ? 2 : 1, s, m->ctx->sm_count));
        }
        PSML_TRY(deal_fork_point(m, s));
        if (l > 0) {
            DealItem *h = find_item(m, l - 1, OP_HADAMARD, 1);
            if (!h) return fail(PSML_ERR_STATE, "missing Hadamard triplet");
            const int64_t w = m->dims[l];
            HadFused<T> hf{};
            for (int p = 0; p < 2; ++p) {
                hf.a[p] = m->tmp.p[p]; hf.b[p] = m->drelu[l - 1].p[p];
                hf.U[p] = h->U.p[p]; hf.V[p] = h->V.p[p]; hf.Z[p] = h->Z.p[p]; hf.c[p] = m->delta.p[p];
            }
            hf.n = B * w;
            hf.em.e[0] = emitB(l - 1, OP_GRADW, B, w);
            hf.em.n = 1;
            if (l - 1 > 0) { hf.em.e[1] = emitA(l - 1, OP_GRADIN, B, w, 0); hf.em.n = 2; }
            ProfScope prof(PROF_HAD, s, 0.0);
            PSML_CUDA_TRY(launch_pdl(had_fused_kernel<T>, dim3(ew_grid(hf.n)), dim3(EW_THREADS), s, hf));
            PSML_LAUNCH_CHECK();
        }
    }
    if (branch) {
        PSML_CUDA_TRY(cudaEventRecord(m->ev_gwj, m->gw));
        PSML_CUDA_TRY(cudaStreamWaitEvent(s, m->ev_gwj, 0));
    }
    return PSML_OK;
}

static psml_status forward_backward(psml_model_s *m, const T *const X[2], const T *const Y[2], cudaStream_t s) {
    if (fused_eligible(m)) return fused_forward_backward(m, X, Y, s);
    PSML_TRY(forward(m, X, Y, nullptr, s));
    return backward(m, s);
}

// ------------------------------------------------------------------------------------------------
// split deployment: one party per process / GPU (include/psml.h "Split deployment").
// The same layer sequence as forward()/backward(), but each opening is an exchange through the
// transport: the party's round kernel writes its masked words to its send buffer, the transport
// delivers the peer's words into the receive buffer laid out identically, and the next kernel
// opens send + recv.  The round kernels are the co-resident ones restricted to party `only`
// (kernels.cuh), so shares and opened values are bit-identical to the co-resident engine.
// ------------------------------------------------------------------------------------------------
static __global__ void add_one_kernel(const T *a, const T *b, int64_t n, T *c) {
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n; e += (int64_t)gridDim.x * blockDim.x)
        c[e] = a[e] + b[e];
}
static __global__ void sub_one_kernel(const T *a, const T *b, int64_t n, T *c) {
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n; e += (int64_t)gridDim.x * blockDim.x)
        c[e] = a[e] - b[e];
}
static __global__ void transpose_one_kernel(const T *in, int64_t R, int64_t C, T *out) {
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < R * C; e += (int64_t)gridDim.x * blockDim.x)
        out[(e % C) * R + e / C] = in[e];
}

struct PartyRun {
    psml_model_s *m;
    int p;            // this party
    psml_xport x;
    cudaStream_t s;
};

struct Msg {
    const T *send;
    T *recv;
    int64_t words;
};
static psml_status xchg(PartyRun &r, std::initializer_list<Msg> msgs) {
    const void *snd[4];
    void *rcv[4];
    int64_t bytes[4];
    int n = 0;
    for (const Msg &b : msgs) {
        snd[n] = b.send; rcv[n] = b.recv; bytes[n] = (int64_t)sizeof(T) * b.words;
        ++n;
    }
    return psml_xport_exchange(r.x, n, snd, rcv, bytes, (psml_stream)r.s);
}

// one party's pair view: slot p = mine, slot 1 - p = nullptr (never touched by `only` kernels)
static inline CPair<T> mine_c(int p, const T *v) {
    CPair<T> c{{nullptr, nullptr}};
    c.p[p] = v;
    return c;
}
static inline Pair<T> mine(int p, T *v) {
    Pair<T> c{{nullptr, nullptr}};
    c.p[p] = v;
    return c;
}

// Beaver product (Eqs. 4-8): mask -> exchange E_i, F_i -> open inside the Eq. 8 GEMM.
static psml_status party_mm(PartyRun &r, const T *A, const T *Bm, int layer, int op, int flags, int trunc, T *C) {
    psml_model_s *m = r.m;
    DealItem *it = find_item(m, layer, op, 0);
    if (!it) return fail(PSML_ERR_STATE, "missing triplet");
    const int64_t M = it->M, K = it->K, N = it->N;
    if (2 * (M * K + K * N) > m->ws_words) return fail(PSML_ERR_STATE, "party workspace too small");
    T *Es = m->ws, *Fs = Es + M * K, *Er = Fs + K * N, *Fr = Er + M * K;
    psml_ctx ctx = reinterpret_cast<psml_ctx>(m->ctx);
    const psml_stream ps = (psml_stream)r.s;
    PSML_TRY(psml_beaver_mask(ctx, r.p, A, Bm, it->U.p[r.p], it->V.p[r.p], M, K, N, flags, Es, Fs, ps));
    PSML_TRY(xchg(r, {{Es, Er, M * K}, {Fs, Fr, K * N}}));
    if (m->d.mask_reuse && op == OP_FWD) {   // keep this layer's openings for the backward products (R26)
        add_one_kernel<<<ew_grid(M * K), EW_THREADS, 0, r.s>>>(Es, Er, M * K, m->eopen[layer]);
        PSML_LAUNCH_CHECK();
        add_one_kernel<<<ew_grid(K * N), EW_THREADS, 0, r.s>>>(Fs, Fr, K * N, m->fopen[layer]);
        PSML_LAUNCH_CHECK();
    }
    return psml_beaver_open_matmul(ctx, r.p, Es, Er, Fs, Fr, it->U.p[r.p], it->V.p[r.p], it->Z.p[r.p], M, K, N, trunc,
                                   C, ps);
}

// Backward products of layer l with mask reuse (R26): ONE exchange (delta_i - D_i); gradW opens to
// (E_f^T, delta) and gradin to (delta, F_f^T) from this party's stored forward openings.
static psml_status party_backward_reuse(PartyRun &r, int l, const T *delta, T *gW, T *gin, int trunc) {
    psml_model_s *m = r.m;
    const int p = r.p;
    DealItem *g = find_item(m, l, OP_GRADW, 0), *gi = l > 0 ? find_item(m, l, OP_GRADIN, 0) : nullptr;
    if (!g || (l > 0 && !gi)) return fail(PSML_ERR_STATE, "missing backward triplet");
    const int64_t B = m->B, din = m->rows[l], dout = m->cols[l];
    psml_ctx ctx = reinterpret_cast<psml_ctx>(m->ctx);
    const psml_stream ps = (psml_stream)r.s;
    sub_one_kernel<<<ew_grid(B * dout), EW_THREADS, 0, r.s>>>(delta, g->V.p[p], B * dout, m->dms);   // delta_i - D_i
    PSML_LAUNCH_CHECK();
    PSML_TRY(xchg(r, {{m->dms, m->dmr, B * dout}}));
    add_one_kernel<<<ew_grid(B * dout), EW_THREADS, 0, r.s>>>(m->dms, m->dmr, B * dout, m->dopen);
    PSML_LAUNCH_CHECK();
    // gradW = A^T . delta: E = E_f^T (din x B), F = delta
    transpose_one_kernel<<<ew_grid(B * din), EW_THREADS, 0, r.s>>>(m->eopen[l], B, din, m->rT);
    PSML_LAUNCH_CHECK();
    PSML_TRY(psml_beaver_open_matmul(ctx, p, m->rT, m->rzero, m->dopen, m->rzero, g->U.p[p], g->V.p[p], g->Z.p[p], din, B,
                                     dout, 0, gW, ps));
    if (!gi) return PSML_OK;
    // gradin = delta . W^T: E = delta, F = F_f^T (dout x din)
    transpose_one_kernel<<<ew_grid(din * dout), EW_THREADS, 0, r.s>>>(m->fopen[l], din, dout, m->rT);
    PSML_LAUNCH_CHECK();
    return psml_beaver_open_matmul(ctx, p, m->dopen, m->rzero, m->rT, m->rzero, gi->U.p[p], gi->V.p[p], gi->Z.p[p], B,
                                   dout, din, trunc, gin, ps);
}

// FSS comparison (R22), one party: round 1 exchanges x_i + r_i, the DCF evaluation gives DReLU,
// round 2 is the Beaver Hadamard x . DReLU.  what 1 = ReLU, 2 = Eq. 9 (x = z of n/2 elements).
static psml_status party_chain_fss(PartyRun &r, const T *x, const DealItem *mat, const DealItem *h, int what, T *y,
                                   T *drelu, const T *Ysub, T *delta) {
    psml_model_s *m = r.m;
    const int p = r.p, q = 1 - p;
    const int64_t n = mat->n;
    T *ws = m->ws;
    T *xin = ws, *d = ws + 3 * n, *rr = ws + 8 * n;
    Pair<T> msg{{nullptr, nullptr}}, mE{{nullptr, nullptr}}, mF{{nullptr, nullptr}};
    msg.p[p] = ws + n; msg.p[q] = ws + 2 * n;
    mE.p[p] = ws + 4 * n; mE.p[q] = ws + 5 * n;
    mF.p[p] = ws + 6 * n; mF.p[q] = ws + 7 * n;
    const T *xe = x;
    if (what == 2) {
        const T half = (T)1 << (m->ctx->ring.frac_bits - 1);
        eq9_prep_kernel<<<ew_grid(n / 2), EW_THREADS, 0, r.s>>>(mine_c(p, x), n / 2, half, mine(p, xin), p);
        PSML_LAUNCH_CHECK();
        xe = xin;
    }
    if (what == 1 && drelu) d = drelu;
    {
        ProfScope prof(PROF_MSB, r.s, 0.0);
        fss_mask_kernel<<<ew_grid(n), EW_THREADS, 0, r.s>>>(mine_c(p, xe), mine_c(p, mat->mat.p[p]), n, msg, p);
        PSML_LAUNCH_CHECK();
    }
    PSML_TRY(xchg(r, {{msg.p[p], msg.p[q], n}}));   // the only opening of the comparison: xhat
    {
        ProfScope prof(PROF_MSB, r.s, 0.0);
        fss_eval_kernel<<<grid_for(n, 128, 148 * 16), 128, 0, r.s>>>(CPair<T>{{msg.p[0], msg.p[1]}},
                                                                    mine_c(p, mat->mat.p[p]), n, mine(p, d), nullptr, p);
        PSML_LAUNCH_CHECK();
    }
    const T *U = h->U.p[p], *V = h->V.p[p], *Z = h->Z.p[p];
    {
        ProfScope prof(PROF_HAD, r.s, 0.0);
        hadamard_mask_kernel<T><<<ew_grid(n), EW_THREADS, 0, r.s>>>(mine_c(p, xe), mine_c(p, d), mine_c(p, U),
                                                                    mine_c(p, V), n, mE, mF, p);
        PSML_LAUNCH_CHECK();
    }
    PSML_TRY(xchg(r, {{mE.p[p], mE.p[q], n}, {mF.p[p], mF.p[q], n}}));
    ProfScope prof(PROF_HAD, r.s, 0.0);
    CPair<T> ce{{mE.p[0], mE.p[1]}}, cf{{mF.p[0], mF.p[1]}};
    hadamard_open_kernel<T><<<ew_grid(n), EW_THREADS, 0, r.s>>>(ce, cf, mine_c(p, U), mine_c(p, V), mine_c(p, Z), n, 0,
                                                               mine(p, what == 2 ? rr : y), p);
    PSML_LAUNCH_CHECK();
    if (what == 2) {
        Pair<T> dl{{nullptr, nullptr}};
        if (delta) dl.p[p] = delta;
        eq9_combine_kernel<<<ew_grid(n / 2), EW_THREADS, 0, r.s>>>(mine_c(p, rr), n / 2, mine(p, y), mine_c(p, Ysub), dl, p);
        PSML_LAUNCH_CHECK();
    }
    return PSML_OK;
}

// MSB chain, one round per kernel with an exchange after each (R9):
// what 1 = ReLU (y = x . drelu, drelu kept), 2 = Eq. 9 (x = z of n/2; y, delta = y - Ysub).
static psml_status party_chain(PartyRun &r, const T *x, const DealItem *mat, const DealItem *h, int what, T *y,
                               T *drelu, const T *Ysub, T *delta) {
    if (mat->kind == IT_FSS) return party_chain_fss(r, x, mat, h, what, y, drelu, Ysub, delta);
    PeerWindow w;
    if (mat->kind == IT_MSB && cur_opts().split_fused && xport_peer_window(r.x, &w)) {
        // one kernel per party: the 9 rounds' exchanges fused over the peer window (split_fused.cuh)
        ChainParty A{};
        A.p = r.p; A.x = x; A.mat = mat->mat.p[r.p];
        A.U = h->U.p[r.p]; A.V = h->V.p[r.p]; A.Z = h->Z.p[r.p];
        A.y = y; A.drelu = drelu; A.Ysub = Ysub; A.delta = delta;
        A.n = mat->n; A.what = what;
        A.half = what == 2 ? (T)1 << (r.m->ctx->ring.frac_bits - 1) : 0;
        A.w = w;
        {
            ProfScope prof(PROF_MSB, r.s, 0.0);
            PSML_TRY(launch_chain_party(A, r.s));
        }
        xport_account(r.x, 9, 17 * 8 * mat->n);
        return PSML_OK;
    }
    psml_model_s *m = r.m;
    const int p = r.p, q = 1 - p;
    const int64_t n = mat->n;
    T *ws = m->ws;
    MsbArgs<T> a;
    a.x = mine_c(p, x);
    a.mat = mine_c(p, mat->mat.p[p]);
    a.G = mine(p, ws + p * n);
    a.P = mine(p, ws + (2 + p) * n);
    a.msg = Pair<T>{{ws + 4 * n, ws + 8 * n}};    // msg.p[p]: my send buffer, msg.p[q]: received
    a.n = n; a.mode = what == 2 ? 1 : 0;
    a.half = what == 2 ? (T)1 << (m->ctx->ring.frac_bits - 1) : (T)0;
    a.l = 64; a.L = 6; a.only = p;
    T *snd = a.msg.p[p], *rcv = a.msg.p[q];
    const int g = ew_grid(n);
    {
        ProfScope prof(PROF_MSB, r.s, 0.0);
        msb_round0_kernel<T><<<g, EW_THREADS, 0, r.s>>>(a);
        PSML_LAUNCH_CHECK();
    }
    PSML_TRY(xchg(r, {{snd, rcv, 2 * n}}));
    for (int j = 1; j <= a.L; ++j) {
        {
            ProfScope prof(PROF_MSB, r.s, 0.0);
            msb_level_kernel<T><<<g, EW_THREADS, 0, r.s>>>(a, j);
            PSML_LAUNCH_CHECK();
        }
        PSML_TRY(xchg(r, {{snd, rcv, 2 * n}}));   // the level's packed G and P AND messages (R27)
    }
    Pair<T> none{{nullptr, nullptr}};
    Pair<T> mE{{a.msg.p[0] + n, a.msg.p[1] + n}}, mF{{a.msg.p[0] + 2 * n, a.msg.p[1] + 2 * n}};
    const T *U = h->U.p[p], *V = h->V.p[p], *Z = h->Z.p[p];
    {
        ProfScope prof(PROF_MSB, r.s, 0.0);
        msb_final_kernel<T><<<g, EW_THREADS, 0, r.s>>>(a, none);
        PSML_LAUNCH_CHECK();
    }
    PSML_TRY(xchg(r, {{snd, rcv, n}}));   // B2A: c_i = msb_i ^ rB_i
    {
        ProfScope prof(PROF_MSB, r.s, 0.0);
        msb_b2a_kernel<T><<<g, EW_THREADS, 0, r.s>>>(a, none, drelu ? mine(p, drelu) : none, mine_c(p, U), mine_c(p, V),
                                                     mE, mF, 1);
        PSML_LAUNCH_CHECK();
    }
    PSML_TRY(xchg(r, {{snd + n, rcv + n, 2 * n}}));   // Hadamard x . drelu: E_i, F_i
    CPair<T> ce{{mE.p[0], mE.p[1]}}, cf{{mF.p[0], mF.p[1]}};
    ProfScope prof(PROF_HAD, r.s, 0.0);
    if (what == 1) {
        hadamard_open_kernel<T><<<g, EW_THREADS, 0, r.s>>>(ce, cf, mine_c(p, U), mine_c(p, V), mine_c(p, Z), n, 0,
                                                           mine(p, y), p);
    } else {
        const int64_t nh = n / 2;
        eq9_open_kernel<T><<<ew_grid(nh), EW_THREADS, 0, r.s>>>(ce, cf, mine_c(p, U), mine_c(p, V), mine_c(p, Z), nh,
                                                                mine(p, y), mine_c(p, Ysub),
                                                                delta ? mine(p, delta) : none, p);
    }
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

// Beaver Hadamard c = a (.) b (untruncated), the backprop DReLU product.
static psml_status party_had(PartyRun &r, const T *a, const T *b, int layer, int slot, T *c) {
    psml_model_s *m = r.m;
    DealItem *h = find_item(m, layer, OP_HADAMARD, slot);
    if (!h) return fail(PSML_ERR_STATE, "missing Hadamard triplet");
    const int p = r.p, q = 1 - p;
    const int64_t n = h->n;
    T *ws = m->ws;
    Pair<T> mE{{ws, ws + n}}, mF{{ws + 2 * n, ws + 3 * n}};
    {
        ProfScope prof(PROF_HAD, r.s, 0.0);
        hadamard_mask_kernel<T><<<ew_grid(n), EW_THREADS, 0, r.s>>>(mine_c(p, a), mine_c(p, b), mine_c(p, h->U.p[p]),
                                                                    mine_c(p, h->V.p[p]), n, mE, mF, p);
        PSML_LAUNCH_CHECK();
    }
    PSML_TRY(xchg(r, {{mE.p[p], mE.p[q], n}, {mF.p[p], mF.p[q], n}}));
    ProfScope prof(PROF_HAD, r.s, 0.0);
    CPair<T> ce{{mE.p[0], mE.p[1]}}, cf{{mF.p[0], mF.p[1]}};
    hadamard_open_kernel<T><<<ew_grid(n), EW_THREADS, 0, r.s>>>(ce, cf, mine_c(p, h->U.p[p]), mine_c(p, h->V.p[p]),
                                                                mine_c(p, h->Z.p[p]), n, 0, mine(p, c), p);
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

// Conv Beaver product (R17): mask the un-expanded input, exchange, open inside the im2col GEMM.
static psml_status party_conv(PartyRun &r, const T *X, const T *Bm, int transposed, int trunc, T *C) {
    psml_model_s *m = r.m;
    DealItem *it = find_item(m, 0, transposed ? OP_GRADW : OP_FWD, 0);
    if (!it) return fail(PSML_ERR_STATE, "missing conv triplet");
    const int64_t nin = m->B * m->g.C * m->g.H * m->g.W, K = it->K, N = it->N;
    T *Es = m->ws, *Fs = Es + nin, *Er = Fs + K * N, *Fr = Er + nin, *partial = Fr + K * N;
    const int64_t pw = m->ws_words - (partial - m->ws);
    if (pw < it->M * N) return fail(PSML_ERR_STATE, "party workspace too small (conv)");
    PSML_TRY(conv_mask_party<T>(X, Bm, it->U.p[r.p], it->V.p[r.p], m->B, m->g, K, N, Es, Fs, r.s));
    PSML_TRY(xchg(r, {{Es, Er, nin}, {Fs, Fr, K * N}}));
    return conv_open_party<T>(r.p, Es, Er, Fs, Fr, it->U.p[r.p], it->V.p[r.p], it->Z.p[r.p], m->B, m->g, transposed,
                              N, trunc, C, partial, pw, r.s, m->ctx->sm_count);
}

static psml_status party_relu(PartyRun &r, const T *x, int layer, T *y, T *dr) {
    DealItem *mat = find_item(r.m, layer, OP_RELU_MSB, 0), *h = find_item(r.m, layer, OP_HADAMARD, 0);
    if (!mat || !h) return fail(PSML_ERR_STATE, "missing ReLU material");
    return party_chain(r, x, mat, h, 1, y, dr, nullptr, nullptr);
}

static psml_status party_cnn(PartyRun &r, const T *X, const T *Y) {
    psml_model_s *m = r.m;
    const int F = m->ctx->ring.frac_bits;
    const int p = r.p;
    m->act[0].p[p] = (T *)X;
    PSML_TRY(party_conv(r, X, m->W[0].p[p], 0, fw(m, 0), m->z[0].p[p]));
    PSML_TRY(party_relu(r, m->z[0].p[p], 0, m->act[1].p[p], m->drelu[0].p[p]));
    PSML_TRY(party_mm(r, m->act[1].p[p], m->W[1].p[p], 1, OP_FWD, 0, fw(m, 1), m->z[1].p[p]));
    PSML_TRY(party_relu(r, m->z[1].p[p], 1, m->act[2].p[p], m->drelu[1].p[p]));
    PSML_TRY(party_mm(r, m->act[2].p[p], m->W[2].p[p], 2, OP_FWD, 0, fw(m, 2), m->z[2].p[p]));
    DealItem *mat = find_item(m, 2, OP_EQ9_MSB, 0), *h = find_item(m, 2, OP_HADAMARD, 2);
    if (!mat || !h) return fail(PSML_ERR_STATE, "missing Eq. 9 material");
    PSML_TRY(party_chain(r, m->z[2].p[p], mat, h, 2, m->yhat.p[p], nullptr, Y, m->delta.p[p]));
    T *g[2];
    PSML_TRY(party_mm(r, m->act[2].p[p], m->delta.p[p], 2, OP_GRADW, PSML_TRANS_A, 0, gradp(m, 2, g)[p]));
    PSML_TRY(party_mm(r, m->delta.p[p], m->W[2].p[p], 2, OP_GRADIN, PSML_TRANS_B, fw(m, 2), m->tmp.p[p]));
    PSML_TRY(party_had(r, m->tmp.p[p], m->drelu[1].p[p], 1, 1, m->delta.p[p]));
    PSML_TRY(party_mm(r, m->act[1].p[p], m->delta.p[p], 1, OP_GRADW, PSML_TRANS_A, 0, gradp(m, 1, g)[p]));
    PSML_TRY(party_mm(r, m->delta.p[p], m->W[1].p[p], 1, OP_GRADIN, PSML_TRANS_B, fw(m, 1), m->tmp.p[p]));
    PSML_TRY(party_had(r, m->tmp.p[p], m->drelu[0].p[p], 0, 1, m->delta.p[p]));
    return party_conv(r, m->act[0].p[p], m->delta.p[p], 1, 0, gradp(m, 0, g)[p]);
}

static psml_status party_forward_backward(PartyRun &r, const T *X, const T *Y) {
    psml_model_s *m = r.m;
    if (m->d.kind == PSML_CNN) return party_cnn(r, X, Y);
    const int F = m->ctx->ring.frac_bits;
    const int p = r.p, nl = m->nl;
    const int64_t B = m->B;
    m->act[0].p[p] = (T *)X;
    for (int l = 0; l < nl; ++l) {
        PSML_TRY(party_mm(r, m->act[l].p[p], m->W[l].p[p], l, OP_FWD, 0, fw(m, l), m->z[l].p[p]));
        if (l < nl - 1) {
            DealItem *mat = find_item(m, l, OP_RELU_MSB, 0), *h = find_item(m, l, OP_HADAMARD, 0);
            if (!mat || !h) return fail(PSML_ERR_STATE, "missing ReLU material");
            PSML_TRY(party_chain(r, m->z[l].p[p], mat, h, 1, m->act[l + 1].p[p], m->drelu[l].p[p], nullptr, nullptr));
        } else if (is_eq9_out(m)) {
            DealItem *mat = find_item(m, l, OP_EQ9_MSB, 0), *h = find_item(m, l, OP_HADAMARD, 2);
            if (!mat || !h) return fail(PSML_ERR_STATE, "missing Eq. 9 material");
            PSML_TRY(party_chain(r, m->z[l].p[p], mat, h, 2, m->yhat.p[p], nullptr, Y, m->delta.p[p]));
        } else {
            const int64_t n = B * m->dims[nl];
            PSML_CUDA_TRY(cudaMemcpyAsync(m->yhat.p[p], m->z[l].p[p], sizeof(T) * n, cudaMemcpyDeviceToDevice, r.s));
            sub_pair_kernel<T><<<ew_grid(n), EW_THREADS, 0, r.s>>>(mine_c(p, m->z[l].p[p]), mine_c(p, Y), n,
                                                                    mine(p, m->delta.p[p]), p);
            PSML_LAUNCH_CHECK();
        }
    }
    T *g[2];
    for (int l = nl - 1; l >= 0; --l) {
        gradp(m, l, g);
        if (m->d.mask_reuse) {
            PSML_TRY(party_backward_reuse(r, l, m->delta.p[p], g[p], m->tmp.p[p], fw(m, l)));
        } else {
            PSML_TRY(party_mm(r, m->act[l].p[p], m->delta.p[p], l, OP_GRADW, PSML_TRANS_A, 0, g[p]));
            if (l > 0)
                PSML_TRY(party_mm(r, m->delta.p[p], m->W[l].p[p], l, OP_GRADIN, PSML_TRANS_B, fw(m, l), m->tmp.p[p]));
        }
        if (l > 0) PSML_TRY(party_had(r, m->tmp.p[p], m->drelu[l - 1].p[p], l - 1, 1, m->delta.p[p]));
    }
    return PSML_OK;
}

}  // namespace psml

using namespace psml;

// ABI definitions: C linkage and default visibility come from include/psml.h.

psml_status psml_model_create(psml_ctx ctx, const psml_model_desc *desc, psml_model *out) {
    PSML_CTX_OPTS(ctx);
    if (!ctx || !desc || !out) return fail(PSML_ERR_INVALID, "null argument");
    Ctx *c = reinterpret_cast<Ctx *>(ctx);
    if (c->ring.l != 64) return fail(PSML_ERR_UNSUPPORTED, "training models run in Z_2^64 (DESIGN.md R18)");
    if (desc->batch <= 0) return fail(PSML_ERR_SHAPE, "batch must be positive");
    if (desc->master_frac_bits < c->ring.frac_bits || desc->lr_shift < 0)
        return fail(PSML_ERR_INVALID, "master_frac_bits must be >= frac_bits and lr_shift >= 0");
    if (2 * c->ring.frac_bits + desc->lr_shift - desc->master_frac_bits < 0)
        return fail(PSML_ERR_INVALID, "2f + lr_shift - m must be >= 0");
    std::unique_ptr<psml_model_s> m(new psml_model_s());
    m->ctx = c;
    m->d = *desc;
    if (desc->deal_role < 0 || desc->deal_role > 2) return fail(PSML_ERR_INVALID, "deal_role must be 0, 1 or 2");
    if (desc->deal_role == 0) m->seeds = dealer_seeds(desc->dealer_seed);           // the dealer: all streams
    else if (desc->deal_role == 1) m->seeds = DealSeeds{0, desc->dealer_seed, 0};   // party 0 holds s_0 only
    else m->seeds = DealSeeds{0, 0, desc->dealer_seed};                             // party 1 holds s_1 only
    m->B = desc->batch;
    switch (desc->kind) {
    case PSML_LINREG:
    case PSML_LOGREG:
    case PSML_SVM:
    case PSML_MLP: {
        int nl = desc->n_layers;
        if (desc->kind != PSML_MLP) nl = 1;
        if (desc->kind == PSML_SVM && desc->dims[1] != 1) return fail(PSML_ERR_SHAPE, "SVM: dims = {d, 1}");
        if (nl < 1 || nl > 7) return fail(PSML_ERR_SHAPE, "n_layers must be in [1, 7]");
        for (int i = 0; i <= nl; ++i)
            if (desc->dims[i] <= 0) return fail(PSML_ERR_SHAPE, "dims must be positive");
        m->nl = nl;
        for (int i = 0; i <= nl; ++i) m->dims.push_back(desc->dims[i]);
        for (int l = 0; l < nl; ++l) { m->rows.push_back(m->dims[l]); m->cols.push_back(m->dims[l + 1]); }
        break;
    }
    case PSML_CNN: {
        ConvGeom g;
        g.C = desc->cnn_c; g.H = desc->cnn_h; g.W = desc->cnn_w; g.k = desc->cnn_k;
        if (g.C <= 0 || g.k <= 0 || g.H < g.k || g.W < g.k || desc->cnn_cout <= 0 || desc->cnn_cout > 16 ||
            desc->cnn_hidden <= 0 || desc->cnn_classes <= 0)
            return fail(PSML_ERR_SHAPE, "bad CNN geometry (cout must be <= 16)");
        g.OH = g.H - g.k + 1; g.OW = g.W - g.k + 1;
        g.coloff = nullptr;
        m->g = g;
        m->nl = 3;
        const int64_t flat = (int64_t)g.OH * g.OW * desc->cnn_cout;
        m->dims = {(int64_t)g.C * g.H * g.W, flat, desc->cnn_hidden, desc->cnn_classes};
        m->rows = {(int64_t)g.C * g.k * g.k, flat, desc->cnn_hidden};
        m->cols = {desc->cnn_cout, desc->cnn_hidden, desc->cnn_classes};
        break;
    }
    case PSML_RNN: {
        const int64_t D = desc->dims[0], H = desc->dims[1], C = desc->dims[2];
        if (D <= 0 || H <= 0 || C <= 0 || desc->rnn_steps <= 0 || desc->rnn_steps > 254)
            return fail(PSML_ERR_SHAPE, "RNN: dims = {D, H, C} > 0 and 1 <= rnn_steps <= 254");
        m->nl = 2;
        m->rnn_T = desc->rnn_steps;
        m->rnn_D = (int)D;
        m->dims = {(int64_t)desc->rnn_steps * D, H, C};
        m->rows = {D + H, H};
        m->cols = {H, C};
        break;
    }
    default:
        return fail(PSML_ERR_INVALID, "unknown model kind");
    }
    if (desc->mask_reuse && desc->kind != PSML_LINREG && desc->kind != PSML_LOGREG && desc->kind != PSML_MLP)
        return fail(PSML_ERR_UNSUPPORTED, "mask_reuse: linear / logistic regression and MLP");
    if (desc->strong_pairs < 0 || desc->strong_pairs > 256) return fail(PSML_ERR_INVALID, "strong_pairs in [0, 256]");
    if (desc->strong_pairs > 1) {   // strong-scaling dealer layout (R28)
        if ((int64_t)desc->pair_id >= desc->strong_pairs) return fail(PSML_ERR_INVALID, "strong scaling: pair_id < strong_pairs");
        if (desc->batch % 8) return fail(PSML_ERR_SHAPE, "strong scaling: batch must be a multiple of 8");
        if (desc->kind == PSML_CNN || desc->mask_reuse)
            return fail(PSML_ERR_UNSUPPORTED, "strong scaling: linear / logistic regression, MLP, SVM, RNN without mask_reuse");
    }
    if (desc->weight_decay_shift < 0 || desc->weight_decay_shift >= 64)
        return fail(PSML_ERR_INVALID, "weight_decay_shift must be in [0, 64)");
    for (int l = 0; l < m->nl; ++l) {
        const int v = desc->fwd_frac_bits[l];
        if (v != 0 && (v < c->ring.frac_bits || v > desc->master_frac_bits))
            return fail(PSML_ERR_INVALID, "fwd_frac_bits must be 0 or in [frac_bits, master_frac_bits]");
    }
    psml_model_s *mp = m.get();
    int64_t tot = 0;
    for (int l = 0; l < m->nl; ++l) {
        Buf b;
        PSML_TRY(balloc(mp, b, m->rows[l] * m->cols[l]));
        m->Wm.push_back(b);
        PSML_TRY(balloc(mp, b, m->rows[l] * m->cols[l]));
        m->W.push_back(b);
        m->grad_off.push_back(tot);
        tot += m->rows[l] * m->cols[l];
    }
    m->grad_words = tot;
    PSML_TRY(dalloc(mp, &m->grad_base, 2 * tot));
    const int64_t B = m->B;
    m->act.resize(m->nl);
    m->z.resize(m->nl);
    m->drelu.resize(m->nl);
    int64_t maxw = 0;
    for (int l = 0; l < m->nl; ++l) {
        if (l >= 1) PSML_TRY(balloc(mp, m->act[l], B * m->dims[l]));
        const int64_t zn = B * m->dims[l + 1];
        PSML_TRY(balloc(mp, m->z[l], zn));
        if (l < m->nl - 1) PSML_TRY(balloc(mp, m->drelu[l], zn));
        maxw = std::max(maxw, std::max(m->dims[l + 1], l >= 1 ? m->dims[l] : (int64_t)0));
    }
    PSML_TRY(balloc(mp, m->yhat, B * m->dims[m->nl]));
    PSML_TRY(balloc(mp, m->delta, B * maxw));
    PSML_TRY(balloc(mp, m->tmp, B * std::max<int64_t>(maxw, 3)));   // SVM: margin, indicator, y (.) ind
    if (m->d.mask_reuse) {
        int64_t mx = 0, bo = 0;
        m->eopen.assign(m->nl, nullptr);
        m->fopen.assign(m->nl, nullptr);
        for (int l = 0; l < m->nl; ++l) {
            PSML_TRY(dalloc(mp, &m->eopen[l], B * m->rows[l]));
            PSML_TRY(dalloc(mp, &m->fopen[l], m->rows[l] * m->cols[l]));
            mx = std::max(mx, std::max(B * m->rows[l], m->rows[l] * m->cols[l]));
            bo = std::max(bo, B * m->cols[l]);
        }
        mx = std::max(mx, bo);
        PSML_TRY(dalloc(mp, &m->dopen, bo));
        PSML_TRY(dalloc(mp, &m->dms, bo));
        PSML_TRY(dalloc(mp, &m->dmr, bo));
        PSML_TRY(dalloc(mp, &m->rT, mx));
        PSML_TRY(dalloc(mp, &m->rzero, mx));
        PSML_CUDA_TRY(cudaMemset(m->rzero, 0, sizeof(T) * mx));
    }
    if (m->d.kind == PSML_RNN) {
        const int64_t T = m->rnn_T, H = m->dims[1];
        PSML_TRY(balloc(mp, m->rnnA, T * B * m->rows[0]));
        PSML_TRY(balloc(mp, m->rnnH, T * B * H));
        PSML_TRY(balloc(mp, m->rnnD, T * B * H));
        PSML_TRY(balloc(mp, m->rnnG, m->rows[0] * H));
    }
    if (m->d.kind == PSML_CNN) {   // im2col column offsets (ch, ky, kx) -> ch*H*W + ky*W + kx
        const ConvGeom &g = m->g;
        std::vector<int32_t> off((size_t)g.C * g.k * g.k);
        for (int ch = 0; ch < g.C; ++ch)
            for (int ky = 0; ky < g.k; ++ky)
                for (int kx = 0; kx < g.k; ++kx) off[(ch * g.k + ky) * g.k + kx] = (ch * g.H + ky) * g.W + kx;
        T *dev = nullptr;
        PSML_TRY(dalloc(mp, &dev, (int64_t)(off.size() + 1) / 2));
        PSML_CUDA_TRY(cudaMemcpy(dev, off.data(), sizeof(int32_t) * off.size(), cudaMemcpyHostToDevice));
        m->g.coloff = (const int32_t *)dev;
    }
    plan_items(mp);
    m->items[1] = m->items[0];
    PSML_TRY(alloc_items(mp, m->items[0]));
    PSML_TRY(alloc_items(mp, m->items[1]));
    for (int pl = 0; pl < 2; ++pl)
        for (int inf = 0; inf < 2; ++inf) PSML_TRY(build_plan(mp, pl, inf != 0));
    if (fused_shapes_ok(mp)) PSML_TRY(alloc_open_bufs(mp));
    m->dws_words = dws_need(mp);
    PSML_TRY(dalloc(mp, &m->dws, m->dws_words));
    {
        // dealer branch at the lowest priority, online branch at the highest: inside the pipelined
        // graph the block scheduler then serves the online kernels first and the dealer's PRG
        // work fills the SMs they leave idle (PSML_PRIO=0 disables)
        int lo = 0, hi = 0;
        PSML_CUDA_TRY(cudaDeviceGetStreamPriorityRange(&lo, &hi));
        // both dealer branches at the lowest priority (raising the first one 1-3 steps measured
        // 900K vs 914K samples/s)
        PSML_CUDA_TRY(cudaStreamCreateWithPriority(&m->side, cudaStreamNonBlocking, lo));
        PSML_CUDA_TRY(cudaStreamCreateWithPriority(&m->side2, cudaStreamNonBlocking, lo));
        PSML_CUDA_TRY(cudaStreamCreateWithPriority(&m->hi, cudaStreamNonBlocking, hi));
        PSML_CUDA_TRY(cudaStreamCreateWithPriority(&m->gw, cudaStreamNonBlocking, hi));
        PSML_CUDA_TRY(cudaStreamCreateWithPriority(&m->d2h, cudaStreamNonBlocking, hi));
        PSML_CUDA_TRY(cudaEventCreateWithFlags(&m->ev_hi, cudaEventDisableTiming));
    }
    PSML_CUDA_TRY(cudaEventCreateWithFlags(&m->ev_fork, cudaEventDisableTiming));
    PSML_CUDA_TRY(cudaEventCreateWithFlags(&m->ev_join, cudaEventDisableTiming));
    PSML_CUDA_TRY(cudaEventCreateWithFlags(&m->ev_late, cudaEventDisableTiming));
    PSML_CUDA_TRY(cudaEventCreateWithFlags(&m->ev_d2, cudaEventDisableTiming));
    PSML_CUDA_TRY(cudaEventCreateWithFlags(&m->ev_gw, cudaEventDisableTiming));
    PSML_CUDA_TRY(cudaEventCreateWithFlags(&m->ev_gwj, cudaEventDisableTiming));
    PSML_CUDA_TRY(cudaEventCreateWithFlags(&m->ev_d2j, cudaEventDisableTiming));
    PSML_CUDA_TRY(cudaEventCreateWithFlags(&m->ev_y, cudaEventDisableTiming));
    PSML_CUDA_TRY(cudaEventCreateWithFlags(&m->ev_yj, cudaEventDisableTiming));
    {
        T *sd = nullptr;
        PSML_TRY(dalloc(mp, &sd, 1));
        m->step_dev = (uint32_t *)sd;
    }
    m->ws_words = ws_need(mp);
    PSML_TRY(dalloc(mp, &m->ws, m->ws_words));
    *out = m.release();
    return PSML_OK;
}

psml_status psml_model_destroy(psml_model model) {
    PSML_CTX_OPTS(model ? model->ctx : nullptr);
    if (!model) return PSML_OK;
    cudaDeviceSynchronize();
    for (int g = 0; g < 2; ++g) {
        if (model->graph[g]) cudaGraphExecDestroy(model->graph[g]);
        if (model->graph_tmpl[g]) cudaGraphDestroy(model->graph_tmpl[g]);
    }
    if (model->side) cudaStreamDestroy(model->side);
    if (model->ev_fork) cudaEventDestroy(model->ev_fork);
    if (model->hi) cudaStreamDestroy(model->hi);
    if (model->ev_hi) cudaEventDestroy(model->ev_hi);
    if (model->ev_join) cudaEventDestroy(model->ev_join);
    if (model->ev_late) cudaEventDestroy(model->ev_late);
    if (model->ev_d2) cudaEventDestroy(model->ev_d2);
    if (model->ev_d2j) cudaEventDestroy(model->ev_d2j);
    if (model->side2) cudaStreamDestroy(model->side2);
    if (model->gw) cudaStreamDestroy(model->gw);
    if (model->ev_gw) cudaEventDestroy(model->ev_gw);
    if (model->ev_gwj) cudaEventDestroy(model->ev_gwj);
    if (model->ev_y) cudaEventDestroy(model->ev_y);
    if (model->ev_yj) cudaEventDestroy(model->ev_yj);
    if (model->d2h) cudaStreamDestroy(model->d2h);
    for (void *p : model->allocs) cudaFree(p);
    delete model;
    return PSML_OK;
}

psml_status psml_model_layer_shape(psml_model m, int32_t layer, int64_t *rows, int64_t *cols) {
    PSML_CTX_OPTS(m ? m->ctx : nullptr);
    if (!m || layer < 0 || layer >= m->nl) return fail(PSML_ERR_INVALID, "bad model or layer");
    if (rows) *rows = m->rows[layer];
    if (cols) *cols = m->cols[layer];
    return PSML_OK;
}

psml_status psml_model_set_master(psml_model m, int32_t layer, const void *const Wm[2], psml_stream stream) {
    PSML_CTX_OPTS(m ? m->ctx : nullptr);
    if (!m || layer < 0 || layer >= m->nl || !Wm) return fail(PSML_ERR_INVALID, "bad model, layer or pointer");
    PSML_TRY(check_ptrs({Wm[0], Wm[1]}));
    cudaStream_t s = (cudaStream_t)stream;
    const int64_t n = m->rows[layer] * m->cols[layer];
    for (int p = 0; p < 2; ++p)
        PSML_CUDA_TRY(cudaMemcpyAsync(m->Wm[layer].p[p], Wm[p], sizeof(T) * n, cudaMemcpyDeviceToDevice, s));
    const int sh = m->d.master_frac_bits - fw(m, layer);
    truncate_pair_kernel<T><<<ew_grid(n), EW_THREADS, 0, s>>>(CPair<T>{{m->Wm[layer].p[0], m->Wm[layer].p[1]}},
                                                               Pair<T>{{m->W[layer].p[0], m->W[layer].p[1]}}, n, sh);
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

psml_status psml_model_get_master(psml_model m, int32_t layer, void *const Wm[2], psml_stream stream) {
    PSML_CTX_OPTS(m ? m->ctx : nullptr);
    if (!m || layer < 0 || layer >= m->nl || !Wm) return fail(PSML_ERR_INVALID, "bad model, layer or pointer");
    PSML_TRY(check_ptrs({Wm[0], Wm[1]}));
    const int64_t n = m->rows[layer] * m->cols[layer];
    for (int p = 0; p < 2; ++p)
        PSML_CUDA_TRY(cudaMemcpyAsync(Wm[p], m->Wm[layer].p[p], sizeof(T) * n, cudaMemcpyDeviceToDevice, (cudaStream_t)stream));
    return PSML_OK;
}

psml_status psml_model_deal(psml_model m, uint32_t step_id, int32_t infer_only, psml_stream stream) {
    PSML_CTX_OPTS(m ? m->ctx : nullptr);
    if (!m) return fail(PSML_ERR_INVALID, "model is null");
    cudaStream_t s = (cudaStream_t)stream;
    const int pool = (int)(step_id & 1);
    set_word_kernel<<<1, 1, 0, s>>>(m->step_dev, step_id);
    PSML_LAUNCH_CHECK();
    m->word_next = -1;
    PSML_TRY(deal_pool(m, pool, step_id, infer_only != 0, s));
    m->dealt_step[pool] = step_id;
    m->dealt_full[pool] = !infer_only;
    return PSML_OK;
}

// Words of party `party`'s material that its own seed cannot produce, in plan order (R23).
static std::vector<std::pair<T *, int64_t>> derived_regions(psml_model_s *m, int pool, int party) {
    std::vector<std::pair<T *, int64_t>> r;
    for (auto &it : m->items[pool]) {
        switch (it.kind) {
        case IT_MATRIX:
        case IT_CONV_FWD:
        case IT_CONV_GW:
        case IT_HAD:
            if (party == 1) r.push_back({it.Z.p[1], it.Z.n});                 // Z_1 = U V - Z_0
            break;
        case IT_MSB:
            if (party == 1) {   // c_1 of the 3 AND groups, r^A_1 of the daBit (R27 layout)
                for (int g = 0; g < 3; ++g) r.push_back({it.mat.p[1] + (3 * (int64_t)g + 2) * it.n, it.n});
                r.push_back({it.mat.p[1] + 10 * it.n, it.n});
            }
            break;
        case IT_FSS:
            r.push_back({it.mat.p[party], (int64_t)FSS_WORDS * it.n});        // DCF keys need both seeds
            break;
        }
    }
    return r;
}

psml_status psml_model_deal_bundle(psml_model m, uint32_t step_id, int32_t party, void *bundle, int64_t *words,
                                   psml_stream stream) {
    PSML_CTX_OPTS(m ? m->ctx : nullptr);
    if (!m || !words) return fail(PSML_ERR_INVALID, "null argument");
    if (party != 0 && party != 1) return fail(PSML_ERR_INVALID, "party must be 0 or 1");
    if (m->d.deal_role != 0) return fail(PSML_ERR_STATE, "only the dealer (deal_role 0) writes bundles");
    const int pool = (int)(step_id & 1);
    int64_t tot = 0;
    for (auto &r : derived_regions(m, pool, party)) tot += r.second;
    *words = tot;
    if (!bundle) return PSML_OK;
    PSML_TRY(check_ptrs({bundle}));
    PSML_TRY(psml_model_deal(m, step_id, 0, stream));
    T *out = (T *)bundle;
    for (auto &r : derived_regions(m, pool, party)) {
        PSML_CUDA_TRY(cudaMemcpyAsync(out, r.first, sizeof(T) * r.second, cudaMemcpyDeviceToDevice, (cudaStream_t)stream));
        out += r.second;
    }
    m->dealt_step[pool] = -1;   // the dealer's own copy is not a party's pool
    return PSML_OK;
}

psml_status psml_model_deal_party(psml_model m, uint32_t step_id, int32_t party, const void *bundle, int64_t words,
                                  psml_stream stream) {
    PSML_CTX_OPTS(m ? m->ctx : nullptr);
    if (!m) return fail(PSML_ERR_INVALID, "model is null");
    if (party != 0 && party != 1) return fail(PSML_ERR_INVALID, "party must be 0 or 1");
    if (m->d.deal_role != party + 1) return fail(PSML_ERR_STATE, "model deal_role is not this party's");
    const int pool = (int)(step_id & 1);
    int64_t tot = 0;
    for (auto &r : derived_regions(m, pool, party)) tot += r.second;
    if (words != tot) return fail(PSML_ERR_SHAPE, "bundle size does not match this model's derived words");
    if (tot && !bundle) return fail(PSML_ERR_INVALID, "bundle is null");
    if (tot) PSML_TRY(check_ptrs({bundle}));
    PSML_TRY(psml_model_deal(m, step_id, 0, stream));   // this party's own streams (the rest is junk)
    const T *in = (const T *)bundle;
    for (auto &r : derived_regions(m, pool, party)) {
        PSML_CUDA_TRY(cudaMemcpyAsync(r.first, in, sizeof(T) * r.second, cudaMemcpyDeviceToDevice, (cudaStream_t)stream));
        in += r.second;
    }
    return PSML_OK;
}

psml_status psml_train_forward_backward(psml_model m, const void *const X[2], const void *const Y[2], uint32_t step_id,
                                        psml_stream stream) {
    PSML_CTX_OPTS(m ? m->ctx : nullptr);
    if (!m || !X || !Y) return fail(PSML_ERR_INVALID, "null argument");
    PSML_TRY(check_ptrs({X[0], X[1], Y[0], Y[1]}));
    const int pool = (int)(step_id & 1);
    if (m->dealt_step[pool] != (int64_t)step_id || !m->dealt_full[pool])
        return fail(PSML_ERR_STATE, "psml_model_deal(step_id, infer_only=0) must precede the step");
    cudaStream_t s = (cudaStream_t)stream;
    m->pool = pool;
    PSML_TRY(forward_backward(m, (const T *const *)X, (const T *const *)Y, s));
    m->dealt_step[pool] = -1;   // the step's material is single-use
    m->grads_ready = true;
    return PSML_OK;
}

psml_status psml_model_output(psml_model m, void **yhat0, void **yhat1, int64_t *n) {
    PSML_CTX_OPTS(m ? m->ctx : nullptr);
    if (!m) return fail(PSML_ERR_INVALID, "model is null");
    if (yhat0) *yhat0 = m->yhat.p[0];
    if (yhat1) *yhat1 = m->yhat.p[1];
    if (n) *n = m->yhat.n;
    return PSML_OK;
}

psml_status psml_model_grads(psml_model m, void **grads, int64_t *words_per_party) {
    PSML_CTX_OPTS(m ? m->ctx : nullptr);
    if (!m) return fail(PSML_ERR_INVALID, "model is null");
    if (grads) *grads = m->grad_base;
    if (words_per_party) *words_per_party = m->grad_words;
    return PSML_OK;
}

psml_status psml_train_apply_update(psml_model m, int32_t extra_shift, psml_stream stream) {
    PSML_CTX_OPTS(m ? m->ctx : nullptr);
    if (!m) return fail(PSML_ERR_INVALID, "model is null");
    if (extra_shift < 0 || extra_shift > 16) return fail(PSML_ERR_INVALID, "extra_shift out of range");
    if (!m->grads_ready) return fail(PSML_ERR_STATE, "no gradients: run psml_train_forward_backward first");
    cudaStream_t s = (cudaStream_t)stream;
    const int f = m->ctx->ring.frac_bits;
    const int s_grad = 2 * f + m->d.lr_shift - m->d.master_frac_bits + extra_shift;
    if (m->nl <= UPD_MAX_LAYERS) {   // every layer in one launch
        UpdateAll<T> u{};
        int64_t tot = 0;
        for (int l = 0; l < m->nl; ++l) {
            T *g[2];
            gradp(m, l, g);
            for (int p = 0; p < 2; ++p) { u.Wm[l][p] = m->Wm[l].p[p]; u.W[l][p] = m->W[l].p[p]; u.g[l][p] = g[p]; }
            u.begin[l] = tot;
            tot += m->rows[l] * m->cols[l];
        }
        u.begin[m->nl] = tot;
        u.nl = m->nl; u.s_grad = s_grad; u.wd = m->d.weight_decay_shift;
        for (int l = 0; l < m->nl; ++l) u.s_fwd[l] = m->d.master_frac_bits - fw(m, l);
        PSML_CUDA_TRY(launch_pdl(update_all_kernel<T>, dim3(ew_grid(tot)), dim3(EW_THREADS), s, u));
        PSML_LAUNCH_CHECK();
        m->grads_ready = false;
        return PSML_OK;
    }
    for (int l = 0; l < m->nl; ++l) {
        const int64_t n = m->rows[l] * m->cols[l];
        T *g[2];
        gradp(m, l, g);
        update_kernel<T><<<ew_grid(n), EW_THREADS, 0, s>>>(Pair<T>{{m->Wm[l].p[0], m->Wm[l].p[1]}},
                                                            Pair<T>{{m->W[l].p[0], m->W[l].p[1]}},
                                                            CPair<T>{{g[0], g[1]}}, n, s_grad,
                                                            m->d.master_frac_bits - fw(m, l), -1,
                                                            m->d.weight_decay_shift);
        PSML_LAUNCH_CHECK();
    }
    m->grads_ready = false;
    return PSML_OK;
}

psml_status psml_secure_train_step(psml_model m, const void *const X[2], const void *const Y[2], uint32_t step_id,
                                   psml_stream stream) {
    PSML_CTX_OPTS(m ? m->ctx : nullptr);
    PSML_TRY(psml_train_forward_backward(m, X, Y, step_id, stream));
    return psml_train_apply_update(m, 0, stream);
}

// The party's data-parallel group: its size n and the update's extra truncation bits -- log2(n)
// when every pair trains its own batch (weak scaling; n = 2^k), 0 under strong scaling (the sum
// over the strong_pairs pairs IS the global-batch gradient, R28)
struct DpGroup {
    psml_status st;
    int32_t n;
    int shift;
};
static DpGroup dp_group(const psml_model_s *m, psml_dp dp) {
    int32_t n = 1;
    if (dp && psml_dp_size(dp, &n) != PSML_OK) return {PSML_ERR_INVALID, 0, 0};
    if (m->d.strong_pairs > 1) {
        if (n != m->d.strong_pairs)
            return {fail(PSML_ERR_INVALID, "strong scaling: the data-parallel group must hold strong_pairs ranks"), n, 0};
        return {PSML_OK, n, 0};
    }
    int sh = 0;
    while ((1 << sh) < n) ++sh;
    if ((1 << sh) != n) return {fail(PSML_ERR_INVALID, "data-parallel group size must be a power of two"), n, 0};
    return {PSML_OK, n, sh};
}

// split deployment: all-reduce this party's untruncated gradient share over its data-parallel
// group, then update its master / forward weight shares
static psml_status party_reduce_update(psml_model_s *m, int party, psml_dp dp, cudaStream_t s) {
    const DpGroup g = dp_group(m, dp);
    PSML_TRY(g.st);
    if (dp && g.n > 1)
        PSML_TRY(psml_dp_allreduce(dp, m->grad_base + (int64_t)party * m->grad_words, m->grad_words, 64, (psml_stream)s));
    return psml_party_apply_update(m, party, g.shift, (psml_stream)s);
}

// One captured step for online pool `pool`.  Non-pipelined: [dealer(pool)] -> online -> [update].
// Pipelined: online(pool) -> [update] on `s`, concurrently dealer(1 - pool) for the NEXT step on the
// side stream (fork/join inside the capture), reading the step word = step + 1.
static bool use_prio() { return true; }   // stream priorities in the pipelined graph (865K -> 914K)

// Client encode + share of a whole minibatch in one launch (psml_model_step_host, Z_2^64): ChaCha20
// blocks [0, nx/8) share X from 8-bit pixels (x = q / 255), the rest share Y from class indices
// (one-hot) or float64 labels -- the same words as psml_encode_share_u8 / _onehot / encode_share.
struct ClientJob {
    PrgKey kx, ky;
    const uint8_t *q;     // X as 8-bit pixels (x = q / 255), or
    const double *xf;     // X as float64 (q == nullptr)
    const uint8_t *ycls;
    const double *yf;
    int64_t nx, ny, classes;
    int f;
    uint64_t *x0, *x1, *y0, *y1;
};
__global__ void __launch_bounds__(128) client_share_kernel(const ClientJob j) {
    const int64_t bx = (j.nx + 7) / 8, total = bx + (j.ny + 7) / 8;
    for (int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; g < total; g += (int64_t)gridDim.x * blockDim.x) {
        const bool isx = g < bx;
        const int64_t b = isx ? g : g - bx, n = isx ? j.nx : j.ny;
        uint32_t w[16];
        chacha20_block(isx ? j.kx : j.ky, (uint32_t)b, w);
#pragma unroll
        for (int t = 0; t < 8; ++t) {
            const int64_t e = b * 8 + t;
            if (e >= n) break;
            double x;
            if (isx) x = j.q ? (double)j.q[e] / 255.0 : j.xf[e];
            else if (j.ycls) x = (int64_t)j.ycls[e / j.classes] == e % j.classes ? 1.0 : 0.0;
            else x = j.yf[e];
            const uint64_t r = ((uint64_t)w[2 * t + 1] << 32) | w[2 * t];
            const uint64_t v = (uint64_t)(unsigned long long)__double2ll_rn(ldexp(x, j.f));
            (isx ? j.x0 : j.y0)[e] = r;
            (isx ? j.x1 : j.y1)[e] = v - r;
        }
    }
}

// out[0..n) = a, out[n..2n) = b (the prediction shares into mapped host memory)
static int64_t x_row(const psml_model_s *m);

// The client's encode + share of the step's batch as the captured graph's first online node
// (co-resident Z_2^64 steps): psml_model_step_device / _host point it at the batch with
// cudaGraphExecKernelNodeSetParams before the replay (no separate launch, no launch gap between
// it and the graph); any other replay sets it to a no-op job (nx = ny = 0).
static ClientJob share_noop(const psml_model_s *m) {
    ClientJob cj{};
    cj.x0 = (T *)m->cap_X[0]; cj.x1 = (T *)m->cap_X[1]; cj.y0 = (T *)m->cap_Y[0]; cj.y1 = (T *)m->cap_Y[1];
    return cj;
}
static psml_status set_share(psml_model_s *m, int g, const ClientJob &cj) {
    cudaKernelNodeParams kp{};
    void *args[1] = {(void *)&cj};
    kp.func = (void *)client_share_kernel;
    kp.gridDim = dim3(m->share_grid);
    kp.blockDim = dim3(128);
    kp.sharedMemBytes = 0;
    kp.kernelParams = args;
    PSML_CUDA_TRY(cudaGraphExecKernelNodeSetParams(m->graph[g], m->share_node[g], &kp));
    return PSML_OK;
}

// the read-back node: both parties' prediction shares (n words each) to out, or a no-op (n = 0)
static psml_status set_out(psml_model_s *m, int g, T *out, int64_t n) {
    cudaKernelNodeParams kp{};
    const T *a = m->yhat.p[0], *b = m->yhat.p[1];
    void *args[4] = {(void *)&a, (void *)&b, (void *)&n, (void *)&out};
    kp.func = (void *)copy_pair_kernel<T>;
    kp.gridDim = dim3(OUT_GRID);
    kp.blockDim = dim3(256);
    kp.sharedMemBytes = 0;
    kp.kernelParams = args;
    PSML_CUDA_TRY(cudaGraphExecKernelNodeSetParams(m->graph[g], m->out_node[g], &kp));
    return PSML_OK;
}

static psml_status capture_one(psml_model_s *m, int pool, const T *const X[2], const T *const Y[2], int flags,
                               cudaStream_t s, cudaGraphExec_t *out, int64_t *kernels, int gi) {
    const bool pipelined = (flags & 4) != 0;
    const bool prio = pipelined && use_prio();
    PSML_CUDA_TRY(cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal));
    psml_status st = PSML_OK;
    cudaStream_t on = s;   // stream of the online phase
    if (pipelined) {
        if (cudaEventRecord(m->ev_fork, s) != cudaSuccess || cudaStreamWaitEvent(m->side, m->ev_fork, 0) != cudaSuccess)
            st = fail(PSML_ERR_CUDA, "graph fork failed");
        if (st == PSML_OK && prio) {
            if (cudaStreamWaitEvent(m->hi, m->ev_fork, 0) != cudaSuccess) st = fail(PSML_ERR_CUDA, "graph fork failed");
            on = m->hi;
        }
        const int after = cur_opts().deal_after;   // default 1: after the step-start open
        // models without the fused step (the CNN) run large kernels that fill the GPU: their
        // dealer forks at the start of the step (measured: 51.6K vs 49.4K samples/s forked after)
        m->deal_after = (fused_eligible(m) && m->cap_party < 0) ? after : 0;
        m->deal_stage = 0;
        m->deal_on_launch = m->deal_after > 0 && cur_opts().deal_on_launch != 0;
        if (m->deal_on_launch) m->deal_after = 2;   // the fork point right after the first product
        m->fork_event_armed = false;
        if (st == PSML_OK && m->deal_after == 0) {
            st = deal_pool(m, 1 - pool, 0, false, m->side, deal_s2(m));
            if (st == PSML_OK) advance_word_kernel<<<1, 1, 0, m->side>>>(m->step_dev);
            if (st == PSML_OK && cudaEventRecord(m->ev_join, m->side) != cudaSuccess)
                st = fail(PSML_ERR_CUDA, "graph join record failed");
        } else {
            m->deal_pending_pool = 1 - pool;   // forked from the online chain (deal_fork_point)
        }
    } else if (flags & 1) {
        st = deal_pool(m, pool, 0, false, s);
    }
    m->pool = pool;
    const int pp = m->cap_party;
    const bool share_node = pp < 0 && m->ctx->ring.l == 64;
    if (st == PSML_OK && share_node) {   // placeholder of the client's share (a no-op until set)
        const int64_t nx = m->B * x_row(m), ny = m->B * m->dims.back();
        m->share_grid = (unsigned)grid_for((nx + 7) / 8 + (ny + 7) / 8, 128);
        ClientJob cj{};
        cj.x0 = (T *)X[0]; cj.x1 = (T *)X[1]; cj.y0 = (T *)Y[0]; cj.y1 = (T *)Y[1];
        client_share_kernel<<<m->share_grid, 128, 0, on>>>(cj);
        if (cudaGetLastError() != cudaSuccess) st = fail(PSML_ERR_CUDA, "share node capture failed");
    }
    m->cap_out = share_node && fused_eligible(m);
    if (st == PSML_OK) {
        if (pp >= 0) {
            PartyRun r{m, pp, m->cap_xport, on};
            st = party_forward_backward(r, X[pp], Y[pp]);
        } else {
            st = forward_backward(m, X, Y, on);
        }
    }
    if (st == PSML_OK && m->cap_out && cudaStreamWaitEvent(on, m->ev_yj, 0) != cudaSuccess)
        st = fail(PSML_ERR_CUDA, "graph join failed");
    const bool out_node = m->cap_out;
    m->cap_out = false;
    if (st == PSML_OK) st = deal_fork_point(m, on, true);   // not forked yet: fork here
    m->deal_pending_pool = -1;
    if (st == PSML_OK && (flags & 2)) {
        m->grads_ready = true;
        st = pp >= 0 ? party_reduce_update(m, pp, m->cap_dp, on) : psml_train_apply_update(m, 0, (psml_stream)on);
    }
    if (prio && st == PSML_OK &&
        (cudaEventRecord(m->ev_hi, m->hi) != cudaSuccess || cudaStreamWaitEvent(s, m->ev_hi, 0) != cudaSuccess))
        st = fail(PSML_ERR_CUDA, "graph join failed");
    if (pipelined && st == PSML_OK && cudaStreamWaitEvent(s, m->ev_join, 0) != cudaSuccess)
        st = fail(PSML_ERR_CUDA, "graph join failed");
    cudaGraph_t g = nullptr;
    cudaError_t e = cudaStreamEndCapture(s, &g);
    if (st != PSML_OK) {
        if (g) cudaGraphDestroy(g);
        return st;
    }
    if (e != cudaSuccess) return fail(PSML_ERR_CUDA, std::string("graph capture: ") + cudaGetErrorString(e));
    size_t nn = 0;
    cudaGraphGetNodes(g, nullptr, &nn);
    std::vector<cudaGraphNode_t> nodes(nn);
    if (nn) cudaGraphGetNodes(g, nodes.data(), &nn);
    *kernels = 0;
    m->share_node[gi] = nullptr;
    m->out_node[gi] = nullptr;
    for (auto nd : nodes) {
        cudaGraphNodeType t;
        if (cudaGraphNodeGetType(nd, &t) == cudaSuccess && t == cudaGraphNodeTypeKernel) {
            ++*kernels;
            cudaKernelNodeParams kp{};
            if ((share_node || out_node) && cudaGraphKernelNodeGetParams(nd, &kp) == cudaSuccess) {
                if (kp.func == (void *)client_share_kernel) m->share_node[gi] = nd;
                if (out_node && kp.func == (void *)copy_pair_kernel<T>) m->out_node[gi] = nd;
            }
        }
    }
    cudaGetLastError();
    // kernel nodes keep the priority of the stream they were captured on
    e = cudaGraphInstantiateWithFlags(out, g, cudaGraphInstantiateFlagUseNodePriority);
    if (e != cudaSuccess) {
        cudaGraphDestroy(g);
        m->share_node[gi] = nullptr;
        m->out_node[gi] = nullptr;
        return fail(PSML_ERR_CUDA, std::string("graph instantiate: ") + cudaGetErrorString(e));
    }
    m->graph_tmpl[gi] = g;   // kept: the share node's handle refers to it
    m->share_live[gi] = false;
    m->out_live[gi] = false;
    return PSML_OK;
}

static psml_status capture_common(psml_model m, const void *const X[2], const void *const Y[2], int32_t flags,
                                  psml_stream stream) {
    if (flags & ~15) return fail(PSML_ERR_INVALID, "flags: bit 0 dealer, bit 1 update, bit 2 pipelined dealer, bit 3 reuse");
    if ((flags & 8) && (flags & 5)) return fail(PSML_ERR_INVALID, "flag bit 3 (material reuse) only applies without a dealer");
    cudaStream_t s = (cudaStream_t)stream;
    if (s == nullptr) return fail(PSML_ERR_INVALID, "capture needs a non-default stream");
    for (int g = 0; g < 2; ++g) {
        if (m->graph[g]) {
            cudaGraphExecDestroy(m->graph[g]);
            m->graph[g] = nullptr;
        }
        if (m->graph_tmpl[g]) {
            cudaGraphDestroy(m->graph_tmpl[g]);
            m->graph_tmpl[g] = nullptr;
        }
        m->share_node[g] = nullptr;
        m->out_node[g] = nullptr;
    }
    const int prof = g_prof_cls.exchange(-1);   // no profiling events inside the graphs
    m->word_next = -1;
    psml_status st = PSML_OK;
    // one graph per dealer pool, except when the graph deals its own pool 0 (flags bit 0 only)
    // or replays one pool on purpose (bit 3, benchmark-only material reuse)
    const bool per_pool = (flags & 4) || !(flags & 9);
    const int ngraphs = per_pool ? 2 : 1;
    for (int g = 0; g < ngraphs && st == PSML_OK; ++g)
        st = capture_one(m, per_pool ? g : 0, (const T *const *)X, (const T *const *)Y, flags, s, &m->graph[g],
                         &m->graph_kernels, g);
    g_prof_cls.store(prof);
    if (st != PSML_OK) return st;
    m->graph_flags = flags;
    for (int i = 0; i < 2; ++i) { m->cap_X[i] = X[i]; m->cap_Y[i] = Y[i]; }
    return PSML_OK;
}

psml_status psml_model_capture_step(psml_model m, const void *const X[2], const void *const Y[2], int32_t flags,
                                   psml_stream stream) {
    PSML_CTX_OPTS(m ? m->ctx : nullptr);
    if (!m || !X || !Y) return fail(PSML_ERR_INVALID, "null argument");
    PSML_TRY(check_ptrs({X[0], X[1], Y[0], Y[1]}));
    m->cap_party = -1;
    m->cap_xport = nullptr;
    m->cap_dp = nullptr;
    return capture_common(m, X, Y, flags, stream);
}

psml_status psml_party_capture_step(psml_model m, int32_t party, psml_xport x, psml_dp dp, const void *X_i,
                                    const void *Y_i, int32_t flags, psml_stream stream) {
    PSML_CTX_OPTS(m ? m->ctx : nullptr);
    if (!m || !x) return fail(PSML_ERR_INVALID, "null model or transport");
    if (party != 0 && party != 1) return fail(PSML_ERR_INVALID, "party must be 0 or 1");
    PSML_TRY(check_ptrs({X_i, Y_i}));
    if (dp) PSML_TRY(dp_group(m, dp).st);
    const void *X[2] = {nullptr, nullptr}, *Y[2] = {nullptr, nullptr};
    X[party] = X_i;
    Y[party] = Y_i;
    m->cap_party = party;
    m->cap_xport = x;
    m->cap_dp = dp;
    const psml_status st = capture_common(m, X, Y, flags, stream);
    if (st != PSML_OK) m->cap_party = -1;
    return st;
}


static psml_status step_graph_job(psml_model_s *m, uint32_t step_id, cudaStream_t s, const ClientJob *job,
                                  T *out, int64_t out_n);

psml_status psml_model_step_host(psml_model m, const uint8_t *q, const void *y, int32_t y_kind, uint64_t share_seed,
                                 uint32_t step_id, void *yhat_host, psml_stream stream) {
    PSML_CTX_OPTS(m ? m->ctx : nullptr);
    if (!m || !q || !y || !yhat_host) return fail(PSML_ERR_INVALID, "null argument");
    if (!m->graph[0] || !m->cap_X[0]) return fail(PSML_ERR_STATE, "no captured step: call psml_model_capture_step first");
    if (y_kind != 0 && y_kind != 1) return fail(PSML_ERR_INVALID, "y_kind: 0 float64 labels, 1 uint8 class indices");
    cudaStream_t s = (cudaStream_t)stream;
    const int64_t nx = m->B * m->dims[0], dl = m->dims.back(), ny = m->B * dl;
    if (!m->stage_q) {
        T *a = nullptr, *b = nullptr;
        PSML_TRY(dalloc(m, &a, (nx + 7) / 8));
        PSML_TRY(dalloc(m, &b, ny));
        m->stage_q = (uint8_t *)a;
        m->stage_y = b;
    }
    // Pinned host buffers mapped into the device address space (cudaHostAlloc / pinned tensors
    // under UVA) are read and written by the kernels directly over PCIe (zero-copy); anything
    // else goes through cudaMemcpyAsync and the device staging buffers.
    auto mapped = [](const void *p) -> void * {
        cudaPointerAttributes a{};
        if (cudaPointerGetAttributes(&a, p) != cudaSuccess) { cudaGetLastError(); return nullptr; }
        return a.type == cudaMemoryTypeHost ? a.devicePointer : nullptr;
    };
    const uint8_t *qd = (const uint8_t *)mapped(q);
    const void *yd = mapped(y);
    T *od = (T *)mapped(yhat_host);
    // client: the compact plaintext batch to the GPU, encode + share into the captured buffers
    if (!qd) {
        PSML_CUDA_TRY(cudaMemcpyAsync(m->stage_q, q, (size_t)nx, cudaMemcpyHostToDevice, s));
        qd = m->stage_q;
    }
    if (!yd) {
        PSML_CUDA_TRY(cudaMemcpyAsync(m->stage_y, y, y_kind ? (size_t)m->B : sizeof(double) * (size_t)ny,
                                      cudaMemcpyHostToDevice, s));
        yd = m->stage_y;
    }
    const psml_ring ring = m->ctx->ring;
    bool shared_in_graph = false, read_in_graph = false;
    const uint64_t cx = call_id(m->d.pair_id, step_id, 0, OP_SHARE, 0), cy = call_id(m->d.pair_id, step_id, 0, OP_SHARE, 1);
    if (ring.l == 64 && nx > 0 && ny > 0) {
        // X and Y in one launch: one PCIe round trip for the mapped host reads instead of two
        ClientJob cj{};
        cj.kx = make_key(share_seed, TAG_SH, cx);
        cj.ky = make_key(share_seed, TAG_SH, cy);
        cj.q = qd; cj.nx = nx; cj.f = ring.frac_bits;
        cj.ycls = y_kind ? (const uint8_t *)yd : nullptr;
        cj.yf = y_kind ? nullptr : (const double *)yd;
        cj.ny = ny; cj.classes = dl;
        cj.x0 = (T *)m->cap_X[0]; cj.x1 = (T *)m->cap_X[1]; cj.y0 = (T *)m->cap_Y[0]; cj.y1 = (T *)m->cap_Y[1];
        if (m->share_node[0]) {   // the graph's own share node: one replay for the whole server side
            read_in_graph = od && m->out_node[0];   // ... and its read-back node, beside the backward pass
            PSML_TRY(step_graph_job(m, step_id, s, &cj, read_in_graph ? od : nullptr, ny));
            shared_in_graph = true;
        } else {
            const int64_t blocks = (nx + 7) / 8 + (ny + 7) / 8;
            client_share_kernel<<<grid_for(blocks, 128), 128, 0, s>>>(cj);
            PSML_LAUNCH_CHECK();
        }
    } else {
        PSML_TRY(psml_encode_share_u8(ring, share_seed, cx, qd, nx, 255.0, (void *)m->cap_X[0], (void *)m->cap_X[1],
                                      stream));
        if (y_kind)
            PSML_TRY(psml_encode_share_onehot(ring, share_seed, cy, (const uint8_t *)yd, m->B, dl, (void *)m->cap_Y[0],
                                              (void *)m->cap_Y[1], stream));
        else
            PSML_TRY(psml_encode_share(ring, share_seed, cy, (const double *)yd, ny, (void *)m->cap_Y[0],
                                       (void *)m->cap_Y[1], stream));
    }
    // servers: the captured step
    if (!shared_in_graph) PSML_TRY(psml_model_step_graph(m, step_id, stream));
    // client: both parties' prediction shares back
    if (read_in_graph) {
        // done by the graph's read-back node
    } else if (od) {
        copy_pair_kernel<T><<<grid_for(2 * ny, 256), 256, 0, s>>>(m->yhat.p[0], m->yhat.p[1], ny, od);
        PSML_LAUNCH_CHECK();
    } else {
        for (int i = 0; i < 2; ++i)
            PSML_CUDA_TRY(cudaMemcpyAsync((uint8_t *)yhat_host + (size_t)i * sizeof(T) * ny, m->yhat.p[i],
                                          sizeof(T) * (size_t)ny, cudaMemcpyDeviceToHost, s));
    }
    return PSML_OK;
}

// features per input row: CNN C H W, RNN T D, else d_0
static int64_t x_row(const psml_model_s *m) {
    if (m->d.kind == PSML_CNN) return (int64_t)m->g.C * m->g.H * m->g.W;
    if (m->d.kind == PSML_RNN) return (int64_t)m->rnn_T * m->rnn_D;
    return m->dims[0];
}

psml_status psml_model_step_device(psml_model m, const double *X, const double *Y, uint64_t share_seed,
                                   uint32_t step_id, psml_stream stream) {
    PSML_CTX_OPTS(m ? m->ctx : nullptr);
    if (!m || !X || !Y) return fail(PSML_ERR_INVALID, "null argument");
    if (!m->graph[0] || !m->cap_X[0]) return fail(PSML_ERR_STATE, "no captured step: call psml_model_capture_step first");
    if (m->cap_party >= 0) return fail(PSML_ERR_STATE, "psml_model_step_device serves the co-resident captured step");
    PSML_TRY(check_ptrs({X, Y}));
    cudaStream_t s = (cudaStream_t)stream;
    const int64_t nx = m->B * x_row(m), ny = m->B * m->dims.back();
    // client: encode + share X and Y into the captured buffers, one launch (R3, R11 share ids)
    ClientJob cj{};
    cj.kx = make_key(share_seed, TAG_SH, call_id(m->d.pair_id, step_id, 0, OP_SHARE, 0));
    cj.ky = make_key(share_seed, TAG_SH, call_id(m->d.pair_id, step_id, 0, OP_SHARE, 1));
    cj.xf = X; cj.nx = nx; cj.f = m->ctx->ring.frac_bits;
    cj.yf = Y; cj.ny = ny; cj.classes = m->dims.back();
    cj.x0 = (T *)m->cap_X[0]; cj.x1 = (T *)m->cap_X[1]; cj.y0 = (T *)m->cap_Y[0]; cj.y1 = (T *)m->cap_Y[1];
    if (m->share_node[0]) return step_graph_job(m, step_id, s, &cj, nullptr, 0);   // the graph's own share node
    client_share_kernel<<<grid_for((nx + 7) / 8 + (ny + 7) / 8, 128), 128, 0, s>>>(cj);
    PSML_LAUNCH_CHECK();
    return psml_model_step_graph(m, step_id, stream);
}

psml_status psml_model_graph_nodes(psml_model m, int64_t *n) {
    PSML_CTX_OPTS(m ? m->ctx : nullptr);
    if (!m || !n) return fail(PSML_ERR_INVALID, "null argument");
    *n = m->graph_kernels;   // (+ a step-word kernel before a replay only when the step sequence jumps)
    return PSML_OK;
}

// One replay of the captured step; job = the client's share of this step's batch for the graph's
// share node (nullptr: the node runs as a no-op).
static psml_status step_graph_job(psml_model_s *m, uint32_t step_id, cudaStream_t s, const ClientJob *job,
                                  T *out = nullptr, int64_t out_n = 0) {
    const bool pipelined = (m->graph_flags & 4) != 0;
    const bool self_dealt = !pipelined && (m->graph_flags & 1);
    const bool reuse = (m->graph_flags & 8) != 0;   // benchmark-only: replays pool 0 as dealt
    const int pool = (self_dealt || reuse) ? 0 : (int)(step_id & 1);
    // A graph without its own dealer consumes material dealt for exactly this step, once: a
    // Beaver mask opened twice on different values would leak their difference.
    if (!self_dealt && !reuse && (m->dealt_step[pool] != (int64_t)step_id || !m->dealt_full[pool]))
        return fail(PSML_ERR_STATE, "psml_model_deal(step_id) must have filled this step's pool (material is single-use)");
    if (reuse && (m->dealt_step[0] < 0 || !m->dealt_full[0]))
        return fail(PSML_ERR_STATE, "reuse graph: pool 0 was never dealt");
    // the step word the graph's dealer reads: a pipelined replay advances it for the next
    // consecutive step itself, so it is written from the host only when the sequence jumps
    const uint32_t word = pipelined ? step_id + 1 : step_id;
    if (!pipelined || m->word_next != (int64_t)word) {
        set_word_kernel<<<1, 1, 0, s>>>(m->step_dev, word);
        PSML_LAUNCH_CHECK();
    }
    const int gi = (self_dealt || reuse) ? 0 : pool;
    if (m->share_node[gi]) {
        if (job) {
            PSML_TRY(set_share(m, gi, *job));
            m->share_live[gi] = true;
        } else if (m->share_live[gi]) {
            PSML_TRY(set_share(m, gi, share_noop(m)));
            m->share_live[gi] = false;
        }
    } else if (job) {
        return fail(PSML_ERR_STATE, "captured step has no share node");
    }
    if (m->out_node[gi]) {
        if (out) {
            PSML_TRY(set_out(m, gi, out, out_n));
            m->out_live[gi] = true;
        } else if (m->out_live[gi]) {
            PSML_TRY(set_out(m, gi, nullptr, 0));
            m->out_live[gi] = false;
        }
    } else if (out) {
        return fail(PSML_ERR_STATE, "captured step has no read-back node");
    }
    PSML_CUDA_TRY(cudaGraphLaunch(m->graph[gi], s));
    m->word_next = pipelined ? (int64_t)word + 1 : -1;
    g_launches.fetch_add((uint64_t)m->graph_kernels);   // the graph's kernels are our launches
    if (pipelined) {
        m->dealt_step[pool] = -1;                        // consumed
        m->dealt_step[1 - pool] = (int64_t)step_id + 1;
        m->dealt_full[1 - pool] = true;
    } else if (self_dealt) {
        m->dealt_step[0] = -1;
    } else if (!reuse) {
        m->dealt_step[pool] = -1;
    }
    m->grads_ready = !(m->graph_flags & 2);
    return PSML_OK;
}

psml_status psml_model_step_graph(psml_model m, uint32_t step_id, psml_stream stream) {
    PSML_CTX_OPTS(m ? m->ctx : nullptr);
    if (!m) return fail(PSML_ERR_INVALID, "model is null");
    if (!m->graph[0]) return fail(PSML_ERR_STATE, "no captured step: call psml_model_capture_step first");
    return step_graph_job(m, step_id, (cudaStream_t)stream, nullptr, nullptr, 0);
}

psml_status psml_secure_infer(psml_model m, const void *const X[2], uint32_t step_id, void *const Yhat[2],
                              psml_stream stream) {
    PSML_CTX_OPTS(m ? m->ctx : nullptr);
    if (!m || !X || !Yhat) return fail(PSML_ERR_INVALID, "null argument");
    PSML_TRY(check_ptrs({X[0], X[1], Yhat[0], Yhat[1]}));
    const int pool = (int)(step_id & 1);
    if (m->dealt_step[pool] != (int64_t)step_id)
        return fail(PSML_ERR_STATE, "psml_model_deal(step_id) must precede inference");
    m->pool = pool;
    PSML_TRY(forward(m, (const T *const *)X, nullptr, (T *const *)Yhat, (cudaStream_t)stream));
    m->dealt_step[pool] = -1;   // the step's material is single-use
    return PSML_OK;
}


// ------------------------------------------------------------------------------------------------
// split deployment ABI
// ------------------------------------------------------------------------------------------------
psml_status psml_party_forward_backward(psml_model m, int32_t party, psml_xport x, const void *X_i, const void *Y_i,
                                        uint32_t step_id, psml_stream stream) {
    PSML_CTX_OPTS(m ? m->ctx : nullptr);
    if (!m || !x) return fail(PSML_ERR_INVALID, "null model or transport");
    if (party != 0 && party != 1) return fail(PSML_ERR_INVALID, "party must be 0 or 1");
    if (m->d.kind == PSML_SVM || m->d.kind == PSML_RNN)
        return fail(PSML_ERR_UNSUPPORTED, "SVM / RNN: co-resident engine only");
    PSML_TRY(check_ptrs({X_i, Y_i}));
    const int pool = (int)(step_id & 1);
    if (m->dealt_step[pool] != (int64_t)step_id || !m->dealt_full[pool])
        return fail(PSML_ERR_STATE, "psml_model_deal(step_id, infer_only=0) must precede the step");
    m->pool = pool;
    PartyRun r{m, party, x, (cudaStream_t)stream};
    PSML_TRY(party_forward_backward(r, (const T *)X_i, (const T *)Y_i));
    m->dealt_step[pool] = -1;   // the step's material is single-use
    m->grads_ready = true;
    return PSML_OK;
}

psml_status psml_party_train_step(psml_model m, int32_t party, psml_xport x, psml_dp dp, const void *X_i,
                                  const void *Y_i, uint32_t step_id, psml_stream stream) {
    PSML_CTX_OPTS(m ? m->ctx : nullptr);
    PSML_TRY(psml_party_forward_backward(m, party, x, X_i, Y_i, step_id, stream));
    if (dp) PSML_TRY(dp_group(m, dp).st);
    return party_reduce_update(m, party, dp, (cudaStream_t)stream);
}

psml_status psml_party_apply_update(psml_model m, int32_t party, int32_t extra_shift, psml_stream stream) {
    PSML_CTX_OPTS(m ? m->ctx : nullptr);
    if (!m) return fail(PSML_ERR_INVALID, "model is null");
    if (party != 0 && party != 1) return fail(PSML_ERR_INVALID, "party must be 0 or 1");
    if (extra_shift < 0 || extra_shift > 16) return fail(PSML_ERR_INVALID, "extra_shift out of range");
    if (!m->grads_ready) return fail(PSML_ERR_STATE, "no gradients: run psml_party_forward_backward first");
    cudaStream_t s = (cudaStream_t)stream;
    const int f = m->ctx->ring.frac_bits;
    const int s_grad = 2 * f + m->d.lr_shift - m->d.master_frac_bits + extra_shift;
    for (int l = 0; l < m->nl; ++l) {
        const int64_t n = m->rows[l] * m->cols[l];
        T *g[2];
        gradp(m, l, g);
        update_kernel<T><<<ew_grid(n), EW_THREADS, 0, s>>>(Pair<T>{{m->Wm[l].p[0], m->Wm[l].p[1]}},
                                                            Pair<T>{{m->W[l].p[0], m->W[l].p[1]}},
                                                            CPair<T>{{g[0], g[1]}}, n, s_grad,
                                                            m->d.master_frac_bits - fw(m, l), party,
                                                            m->d.weight_decay_shift);
        PSML_LAUNCH_CHECK();
    }
    m->grads_ready = false;
    return PSML_OK;
}
