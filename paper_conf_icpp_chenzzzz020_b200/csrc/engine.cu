// engine.cu -- the C ABI of include/psml.h: context, client/dealer calls, secure ops.
// Models / training live in model.cu.
#include <cstdio>
#include <cstring>
#include <mutex>
#include <string>
#include <utility>
#include <vector>

#include "engine.h"
#include "fss.cuh"

namespace psml {

static thread_local std::string g_err;
std::atomic<uint64_t> g_launches{0};

std::atomic<int> g_prof_cls{-1};
static std::mutex g_prof_mu;
static std::vector<std::pair<cudaEvent_t, cudaEvent_t>> g_prof_pairs;
static std::vector<cudaEvent_t> g_prof_pool;
static double g_prof_work = 0;

cudaEvent_t prof_event() {
    std::lock_guard<std::mutex> lk(g_prof_mu);
    if (!g_prof_pool.empty()) {
        cudaEvent_t e = g_prof_pool.back();
        g_prof_pool.pop_back();
        return e;
    }
    cudaEvent_t e = nullptr;
    cudaEventCreate(&e);
    return e;
}

void prof_record(cudaEvent_t a, cudaEvent_t b, double work) {
    std::lock_guard<std::mutex> lk(g_prof_mu);
    g_prof_pairs.emplace_back(a, b);
    g_prof_work += work;
}

void set_error(const std::string &msg) { g_err = msg; }
psml_status fail(psml_status st, const std::string &msg) {
    g_err = msg;
    return st;
}

int current_sm_count() {
    int dev = 0, sms = 148;
    if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    return sms;
}

psml_status check_ring(psml_ring r) {
    if (r.l != 32 && r.l != 64) return fail(PSML_ERR_INVALID, "ring.l must be 32 or 64");
    if (r.frac_bits < 0 || r.frac_bits >= r.l) return fail(PSML_ERR_INVALID, "ring.frac_bits out of range");
    return PSML_OK;
}

psml_status check_ptrs(std::initializer_list<const void *> ps) {
    for (const void *p : ps) {
        if (p == nullptr) return fail(PSML_ERR_INVALID, "null device pointer");
        if (!aligned16(p)) return fail(PSML_ERR_ALIGN, "pointer not 16-byte aligned");
    }
    return PSML_OK;
}

psml_status Ctx::ensure_ws(size_t bytes) {
    if (bytes <= ws_bytes) return PSML_OK;
    if (ws) {
        PSML_CUDA_TRY(cudaDeviceSynchronize());
        PSML_CUDA_TRY(cudaFree(ws));
        ws = nullptr;
        ws_bytes = 0;
    }
    size_t want = std::max(bytes, (size_t)1 << 20);
    if (cudaMalloc(&ws, want) != cudaSuccess) {
        cudaGetLastError();
        return fail(PSML_ERR_NOMEM, "workspace allocation of " + std::to_string(want) + " bytes failed");
    }
    ws_bytes = want;
    return PSML_OK;
}

}  // namespace psml

using namespace psml;

// ABI definitions: C linkage and default visibility come from include/psml.h.

int32_t psml_abi_version(void) { return PSML_ABI_VERSION; }
const char *psml_last_error(void) { return g_err.c_str(); }
uint64_t psml_kernel_launch_count(void) { return g_launches.load(); }

psml_status psml_prof_enable(int32_t cls) {
    if (cls < -1 || cls > 5) return fail(PSML_ERR_INVALID, "profile class must be in [-1, 5]");
    g_prof_cls.store(cls);
    return PSML_OK;
}

psml_status psml_prof_read(double *total_ms, int64_t *launches, double *work) {
    PSML_CUDA_TRY(cudaDeviceSynchronize());
    std::lock_guard<std::mutex> lk(g_prof_mu);
    double ms = 0;
    for (auto &pr : g_prof_pairs) {
        float t = 0;
        if (cudaEventElapsedTime(&t, pr.first, pr.second) == cudaSuccess) ms += t;
        g_prof_pool.push_back(pr.first);
        g_prof_pool.push_back(pr.second);
    }
    if (total_ms) *total_ms = ms;
    if (launches) *launches = (int64_t)g_prof_pairs.size();
    if (work) *work = g_prof_work;
    g_prof_pairs.clear();
    g_prof_work = 0;
    return PSML_OK;
}

// Ring multiply-add throughput microbenchmark (the ALU roofline denominator of the CUDA-core ring
// GEMMs): 8 independent accumulator chains per thread of acc = acc + a * b in
// Z_2^64 (IMAD.WIDE.U32 + 2 IMAD, the GEMM inner loop's mix) or Z_2^32 (one IMAD).
template <typename T>
__global__ void __launch_bounds__(256) mac_peak_kernel(T a0, T b0, int iters, T *out) {
    T acc[8], a[8];
    const T b = b0 + (T)threadIdx.x;
#pragma unroll
    for (int j = 0; j < 8; ++j) { acc[j] = (T)(blockIdx.x * 8 + j); a[j] = a0 + (T)(j * 0x9E3779B9u) + (T)threadIdx.x; }
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int j = 0; j < 8; ++j) acc[j] = acc[j] + a[j] * b;
#pragma unroll
        for (int j = 0; j < 8; ++j) a[j] = acc[j];   // chain through memory-free dependencies
    }
    T r = 0;
#pragma unroll
    for (int j = 0; j < 8; ++j) r ^= acc[j];
    if (r == (T)0x1234567) out[0] = r;   // keeps the loop alive
}

psml_status psml_bench_mac_peak(int32_t l, double *ring_macs_per_s) {
    if ((l != 32 && l != 64) || !ring_macs_per_s) return fail(PSML_ERR_INVALID, "l must be 32 or 64");
    int dev = 0, sms = 0;
    PSML_CUDA_TRY(cudaGetDevice(&dev));
    PSML_CUDA_TRY(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    void *out = nullptr;
    PSML_CUDA_TRY(cudaMalloc(&out, 8));
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const int blocks = sms * 8, iters = 4096;
    float best = 1e30f;
    for (int rep = 0; rep < 4; ++rep) {
        cudaEventRecord(e0);
        if (l == 64) mac_peak_kernel<uint64_t><<<blocks, 256>>>(0x1234567890ull, 0x9E3779B97F4A7C15ull, iters, (uint64_t *)out);
        else mac_peak_kernel<uint32_t><<<blocks, 256>>>(0x12345u, 0x9E3779B9u, iters, (uint32_t *)out);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms = 0;
        cudaEventElapsedTime(&ms, e0, e1);
        if (rep > 0) best = std::min(best, ms);
    }
    const cudaError_t e = cudaGetLastError();
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(out);
    if (e != cudaSuccess) return fail(PSML_ERR_CUDA, cudaGetErrorString(e));
    *ring_macs_per_s = (double)blocks * 256 * iters * 8 / (best * 1e-3);
    return PSML_OK;
}

namespace psml {
// Host ChaCha20 block (RFC 8439 Sec. 2.3), used only to derive the parties' dealer seeds.
static void host_chacha20(const uint32_t key[8], uint32_t counter, const uint32_t nonce[3], uint32_t out[16]) {
    auto rl = [](uint32_t v, int c) { return (v << c) | (v >> (32 - c)); };
    uint32_t st[16] = {0x61707865u, 0x3320646eu, 0x79622d32u, 0x6b206574u, key[0], key[1], key[2], key[3],
                       key[4],      key[5],      key[6],      key[7],      counter, nonce[0], nonce[1], nonce[2]};
    uint32_t x[16];
    for (int i = 0; i < 16; ++i) x[i] = st[i];
    auto qr = [&](int a, int b, int c, int d) {
        x[a] += x[b]; x[d] ^= x[a]; x[d] = rl(x[d], 16);
        x[c] += x[d]; x[b] ^= x[c]; x[b] = rl(x[b], 12);
        x[a] += x[b]; x[d] ^= x[a]; x[d] = rl(x[d], 8);
        x[c] += x[d]; x[b] ^= x[c]; x[b] = rl(x[b], 7);
    };
    for (int r = 0; r < 10; ++r) {
        qr(0, 4, 8, 12); qr(1, 5, 9, 13); qr(2, 6, 10, 14); qr(3, 7, 11, 15);
        qr(0, 5, 10, 15); qr(1, 6, 11, 12); qr(2, 7, 8, 13); qr(3, 4, 9, 14);
    }
    for (int i = 0; i < 16; ++i) out[i] = x[i] + st[i];
}

// s_i = element 0 of the PRG stream (dealer seed, "KD", call id i)  (R1, R23)
static uint64_t party_seed(uint64_t dealer_seed, int party) {
    const uint32_t key[8] = {(uint32_t)dealer_seed, (uint32_t)(dealer_seed >> 32), 0, 0, 0, 0, 0, 0};
    const uint32_t nonce[3] = {0x0000444Bu /* "KD" */, (uint32_t)party, 0};
    uint32_t w[16];
    host_chacha20(key, 0, nonce, w);
    return ((uint64_t)w[1] << 32) | w[0];
}

DealSeeds dealer_seeds(uint64_t dealer_seed) { return DealSeeds{dealer_seed, party_seed(dealer_seed, 0), party_seed(dealer_seed, 1)}; }
}  // namespace psml

uint64_t psml_dealer_party_seed(uint64_t dealer_seed, int32_t party) {
    return (party == 0 || party == 1) ? party_seed(dealer_seed, party) : 0;
}

psml_status psml_device_info(int32_t *sm_count, int32_t *cc_major, int32_t *cc_minor) {
    int dev = 0, n = 0;
    if (cudaGetDeviceCount(&n) != cudaSuccess || n == 0) {
        cudaGetLastError();
        return fail(PSML_ERR_UNSUPPORTED, "no CUDA device visible");
    }
    PSML_CUDA_TRY(cudaGetDevice(&dev));
    int a = 0, b = 0, c = 0;
    PSML_CUDA_TRY(cudaDeviceGetAttribute(&a, cudaDevAttrMultiProcessorCount, dev));
    PSML_CUDA_TRY(cudaDeviceGetAttribute(&b, cudaDevAttrComputeCapabilityMajor, dev));
    PSML_CUDA_TRY(cudaDeviceGetAttribute(&c, cudaDevAttrComputeCapabilityMinor, dev));
    if (sm_count) *sm_count = a;
    if (cc_major) *cc_major = b;
    if (cc_minor) *cc_minor = c;
    return PSML_OK;
}

psml_status psml_ctx_create(psml_ring ring, int32_t gemm_backend, psml_ctx *out) {
    PSML_TRY(check_ring(ring));
    if (!out) return fail(PSML_ERR_INVALID, "out is null");
    if (gemm_backend < 0 || gemm_backend > 2) return fail(PSML_ERR_INVALID, "gemm_backend must be 0, 1 or 2");
    int32_t sms = 0, maj = 0, mnr = 0;
    PSML_TRY(psml_device_info(&sms, &maj, &mnr));
    if (gemm_backend == 2 && !(maj == 10 && mnr == 0))
        return fail(PSML_ERR_UNSUPPORTED, "tcgen05 backend needs an sm_100 device");
    Ctx *c = new Ctx();
    c->ring = ring;
    c->backend = gemm_backend;
    c->sm_count = sms;
    c->tc_ok = (maj == 10 && mnr == 0);
    *out = reinterpret_cast<psml_ctx>(c);
    return PSML_OK;
}

psml_status Ctx::ensure_msg(size_t bytes) {
    if (bytes <= msg_bytes) return PSML_OK;
    if (msg) {
        PSML_CUDA_TRY(cudaDeviceSynchronize());
        PSML_CUDA_TRY(cudaFree(msg));
        msg = nullptr;
        msg_bytes = 0;
    }
    if (cudaMalloc(&msg, bytes) != cudaSuccess) {
        cudaGetLastError();
        return fail(PSML_ERR_NOMEM, "message buffer allocation failed");
    }
    msg_bytes = bytes;
    return PSML_OK;
}

psml_status psml_ctx_create_party(psml_ring ring, int32_t gemm_backend, int32_t party, psml_xport pair, psml_dp dp,
                                  psml_ctx *out) {
    if (party != 0 && party != 1) return fail(PSML_ERR_INVALID, "party must be 0 or 1");
    if (!pair) return fail(PSML_ERR_INVALID, "a per-party context needs its pair transport");
    PSML_TRY(psml_ctx_create(ring, gemm_backend, out));
    Ctx *c = reinterpret_cast<Ctx *>(*out);
    c->party = party;
    c->xport = pair;
    c->dp = dp;
    return PSML_OK;
}

psml_status psml_secure_matmul_party(psml_ctx ctx, const void *A_i, const void *B_i, const void *U_i, const void *V_i,
                                     const void *Z_i, int64_t M, int64_t K, int64_t N, int32_t flags,
                                     int32_t trunc_bits, void *C_i, psml_stream stream) {
    PSML_CTX_OPTS(ctx);
    if (!ctx) return fail(PSML_ERR_INVALID, "ctx is null");
    Ctx *c = reinterpret_cast<Ctx *>(ctx);
    if (c->party < 0 || !c->xport) return fail(PSML_ERR_STATE, "not a per-party context (psml_ctx_create_party)");
    if (M <= 0 || K <= 0 || N <= 0) return fail(PSML_ERR_SHAPE, "M, K, N must be positive");
    const size_t w = c->ring.l / 8;
    auto up = [](size_t x) { return (x + 255) & ~(size_t)255; };   // 16-byte aligned sub-buffers
    const size_t eb = up(w * M * K), fb = up(w * K * N);
    PSML_TRY(c->ensure_msg(2 * (eb + fb)));
    uint8_t *b = (uint8_t *)c->msg;
    void *Es = b, *Fs = b + eb, *Er = b + eb + fb, *Fr = b + 2 * eb + fb;
    // round 1 (Eq. 4), the exchange of E_i and F_i (Eq. 5) through the pair transport, round 2
    PSML_TRY(psml_beaver_mask(ctx, c->party, A_i, B_i, U_i, V_i, M, K, N, flags, Es, Fs, stream));
    const void *snd[2] = {Es, Fs};
    void *rcv[2] = {Er, Fr};
    const int64_t bytes[2] = {(int64_t)w * M * K, (int64_t)w * K * N};
    PSML_TRY(psml_xport_exchange(c->xport, 2, snd, rcv, bytes, stream));
    return psml_beaver_open_matmul(ctx, c->party, Es, Er, Fs, Fr, U_i, V_i, Z_i, M, K, N, trunc_bits, C_i, stream);
}

namespace psml {
static const psml_options k_default_opts{0, 1, 0, 1, 1, 1, 1, 1, 1, 1, 0, 1, 1, 0, 1};
static thread_local const psml_options *t_opts = nullptr;
static thread_local cudaEvent_t t_launch_event = nullptr;
void arm_launch_event(cudaEvent_t e) { t_launch_event = e; }
cudaEvent_t take_launch_event() {
    cudaEvent_t e = t_launch_event;
    t_launch_event = nullptr;
    return e;
}
const psml_options &cur_opts() { return t_opts ? *t_opts : k_default_opts; }
OptScope::OptScope(const psml_options *o) : prev(t_opts) { if (o) t_opts = o; }
OptScope::~OptScope() { t_opts = prev; }
}  // namespace psml

psml_status psml_options_default(psml_options *out) {
    if (!out) return fail(PSML_ERR_INVALID, "out is null");
    *out = k_default_opts;
    return PSML_OK;
}

psml_status psml_ctx_set_options(psml_ctx ctx, const psml_options *o) {
    if (!ctx || !o) return fail(PSML_ERR_INVALID, "null argument");
    if (o->seg_backend < 0 || o->seg_backend > 2 || o->msb_chain < 0 || o->msb_chain > 1 || o->deal_after < 0 ||
        o->deal_on_launch < 0 || o->deal_on_launch > 1 || o->tc_small < 0 || o->tc_small > 2)
        return fail(PSML_ERR_INVALID, "option out of range");
    reinterpret_cast<Ctx *>(ctx)->opts = *o;
    return PSML_OK;
}

psml_status psml_ctx_destroy(psml_ctx ctx) {
    if (!ctx) return PSML_OK;
    Ctx *c = reinterpret_cast<Ctx *>(ctx);
    if (c->ws || c->msg) cudaDeviceSynchronize();
    if (c->msg) cudaFree(c->msg);
    if (c->ws) {
        cudaFree(c->ws);
    }
    delete c;
    return PSML_OK;
}

// ------------------------------------------------------------------------------------------------
// client side
// ------------------------------------------------------------------------------------------------
psml_status psml_prg_fill(psml_ring ring, uint64_t seed, uint32_t tag, uint64_t call_id, uint64_t offset,
                          int64_t n, void *out, psml_stream stream) {
    PSML_TRY(check_ring(ring));
    if (n < 0) return fail(PSML_ERR_SHAPE, "n < 0");
    if (n == 0) return PSML_OK;
    PSML_TRY(check_ptrs({out}));
    cudaStream_t s = (cudaStream_t)stream;
    PrgKey k = make_key(seed, tag, call_id);
    const int64_t nblk = n / (ring.l == 64 ? 8 : 16) + 2;
    if (ring.l == 64) prg_kernel<uint64_t, 0><<<grid_for(nblk, 256), 256, 0, s>>>(k, offset, n, (uint64_t *)out, nullptr, nullptr);
    else prg_kernel<uint32_t, 0><<<grid_for(nblk, 256), 256, 0, s>>>(k, offset, n, (uint32_t *)out, nullptr, nullptr);
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

psml_status psml_encode(psml_ring ring, const double *x, int64_t n, void *v, psml_stream stream) {
    PSML_TRY(check_ring(ring));
    if (n < 0) return fail(PSML_ERR_SHAPE, "n < 0");
    if (n == 0) return PSML_OK;
    PSML_TRY(check_ptrs({x, v}));
    cudaStream_t s = (cudaStream_t)stream;
    if (ring.l == 64) encode_kernel<uint64_t><<<grid_for(n, 256), 256, 0, s>>>(x, n, ring.frac_bits, (uint64_t *)v);
    else encode_kernel<uint32_t><<<grid_for(n, 256), 256, 0, s>>>(x, n, ring.frac_bits, (uint32_t *)v);
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

psml_status psml_decode(psml_ring ring, const void *v, int64_t n, double *x, psml_stream stream) {
    PSML_TRY(check_ring(ring));
    if (n < 0) return fail(PSML_ERR_SHAPE, "n < 0");
    if (n == 0) return PSML_OK;
    PSML_TRY(check_ptrs({x, v}));
    cudaStream_t s = (cudaStream_t)stream;
    if (ring.l == 64) decode_kernel<uint64_t><<<grid_for(n, 256), 256, 0, s>>>((const uint64_t *)v, n, ring.frac_bits, x);
    else decode_kernel<uint32_t><<<grid_for(n, 256), 256, 0, s>>>((const uint32_t *)v, n, ring.frac_bits, x);
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

psml_status psml_share(psml_ring ring, uint64_t seed, uint64_t stream_id, const void *x, int64_t n, void *x0,
                       void *x1, psml_stream stream) {
    PSML_TRY(check_ring(ring));
    if (n < 0) return fail(PSML_ERR_SHAPE, "n < 0");
    if (n == 0) return PSML_OK;
    PSML_TRY(check_ptrs({x, x0, x1}));
    if (x == x0 || x == x1 || x0 == x1) return fail(PSML_ERR_INVALID, "share outputs must not alias the input");
    cudaStream_t s = (cudaStream_t)stream;
    PrgKey k = make_key(seed, TAG_SH, stream_id);
    const int64_t nblk = n / (ring.l == 64 ? 8 : 16) + 2;
    if (ring.l == 64)
        prg_kernel<uint64_t, 1><<<grid_for(nblk, 256), 256, 0, s>>>(k, 0, n, (uint64_t *)x0, (const uint64_t *)x, (uint64_t *)x1);
    else
        prg_kernel<uint32_t, 1><<<grid_for(nblk, 256), 256, 0, s>>>(k, 0, n, (uint32_t *)x0, (const uint32_t *)x, (uint32_t *)x1);
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

psml_status psml_encode_share(psml_ring ring, uint64_t seed, uint64_t stream_id, const double *x, int64_t n,
                              void *x0, void *x1, psml_stream stream) {
    PSML_TRY(check_ring(ring));
    if (n < 0) return fail(PSML_ERR_SHAPE, "n < 0");
    if (n == 0) return PSML_OK;
    PSML_TRY(check_ptrs({x, x0, x1}));
    if (x0 == x1) return fail(PSML_ERR_INVALID, "share outputs must not alias");
    cudaStream_t s = (cudaStream_t)stream;
    PrgKey k = make_key(seed, TAG_SH, stream_id);
    const int64_t nblk = n / (ring.l == 64 ? 8 : 16) + 1;
    if (ring.l == 64)
        encode_share_kernel<uint64_t><<<grid_for(nblk, 128), 128, 0, s>>>(k, n, ring.frac_bits, x, (uint64_t *)x0,
                                                                           (uint64_t *)x1);
    else
        encode_share_kernel<uint32_t><<<grid_for(nblk, 128), 128, 0, s>>>(k, n, ring.frac_bits, x, (uint32_t *)x0,
                                                                           (uint32_t *)x1);
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

static psml_status encode_share_u8(psml_ring ring, uint64_t seed, uint64_t stream_id, const uint8_t *q, int64_t n,
                                   double den, int64_t classes, void *x0, void *x1, psml_stream stream) {
    PSML_TRY(check_ring(ring));
    if (n < 0) return fail(PSML_ERR_SHAPE, "n < 0");
    if (n == 0) return PSML_OK;
    PSML_TRY(check_ptrs({q, x0, x1}));
    if (x0 == x1) return fail(PSML_ERR_INVALID, "share outputs must not alias");
    cudaStream_t s = (cudaStream_t)stream;
    PrgKey k = make_key(seed, TAG_SH, stream_id);
    const int64_t nblk = n / (ring.l == 64 ? 8 : 16) + 1;
    if (ring.l == 64)
        encode_share_u8_kernel<uint64_t><<<grid_for(nblk, 128), 128, 0, s>>>(k, n, ring.frac_bits, q, den, classes,
                                                                              (uint64_t *)x0, (uint64_t *)x1);
    else
        encode_share_u8_kernel<uint32_t><<<grid_for(nblk, 128), 128, 0, s>>>(k, n, ring.frac_bits, q, den, classes,
                                                                              (uint32_t *)x0, (uint32_t *)x1);
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

psml_status psml_encode_share_u8(psml_ring ring, uint64_t seed, uint64_t stream_id, const uint8_t *q, int64_t n,
                                 double den, void *x0, void *x1, psml_stream stream) {
    if (!(den > 0.0)) return fail(PSML_ERR_INVALID, "den must be > 0");
    return encode_share_u8(ring, seed, stream_id, q, n, den, 1, x0, x1, stream);
}

psml_status psml_encode_share_onehot(psml_ring ring, uint64_t seed, uint64_t stream_id, const uint8_t *cls,
                                     int64_t rows, int64_t classes, void *x0, void *x1, psml_stream stream) {
    if (rows < 0 || classes <= 0) return fail(PSML_ERR_SHAPE, "rows < 0 or classes <= 0");
    return encode_share_u8(ring, seed, stream_id, cls, rows * classes, 0.0, classes, x0, x1, stream);
}

psml_status psml_reconstruct(psml_ring ring, const void *x0, const void *x1, int64_t n, void *x,
                             psml_stream stream) {
    PSML_TRY(check_ring(ring));
    if (n < 0) return fail(PSML_ERR_SHAPE, "n < 0");
    if (n == 0) return PSML_OK;
    PSML_TRY(check_ptrs({x0, x1, x}));
    cudaStream_t s = (cudaStream_t)stream;
    if (ring.l == 64) add_kernel<uint64_t><<<grid_for(n, 256), 256, 0, s>>>((const uint64_t *)x0, (const uint64_t *)x1, n, (uint64_t *)x);
    else add_kernel<uint32_t><<<grid_for(n, 256), 256, 0, s>>>((const uint32_t *)x0, (const uint32_t *)x1, n, (uint32_t *)x);
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

// ------------------------------------------------------------------------------------------------
// dealer
// ------------------------------------------------------------------------------------------------
// rows [row0, row0 + M) of the triplet (row0 = 0: the whole M x K by K x N triplet)
template <typename T>
static psml_status triplet_gen_t(Ctx *c, uint64_t seed, uint64_t cid, int64_t row0, int64_t M, int64_t K, int64_t N,
                                 void *const U[2], void *const V[2], void *const Z[2], cudaStream_t s) {
    const DealSeeds S = dealer_seeds(seed);
    if (row0 == 0) {
        dealer_pair_kernel<T><<<grid_for(M * K / 8 + 1, 256), 256, 0, s>>>(dkey(S, TAG_U0, cid), dkey(S, TAG_U1, cid),
                                                                           M * K, (T *)U[0], (T *)U[1], nullptr);
        PSML_LAUNCH_CHECK();
    } else {   // a row block: the U streams from element row0 * K (any alignment)
        for (int i = 0; i < 2; ++i) {
            prg_kernel<T, 0><<<grid_for(M * K / 8 + 2, 256), 256, 0, s>>>(dkey(S, i ? TAG_U1 : TAG_U0, cid), row0 * K,
                                                                          M * K, (T *)U[i], nullptr, nullptr);
            PSML_LAUNCH_CHECK();
        }
    }
    dealer_pair_kernel<T><<<grid_for(K * N / 8 + 1, 256), 256, 0, s>>>(dkey(S, TAG_V0, cid), dkey(S, TAG_V1, cid), K * N,
                                                                       (T *)V[0], (T *)V[1], nullptr);
    PSML_LAUNCH_CHECK();
    prg_kernel<T, 0><<<grid_for(M * N / 8 + 2, 256), 256, 0, s>>>(dkey(S, TAG_Z0, cid), row0 * N, M * N, (T *)Z[0],
                                                                  nullptr, nullptr);
    PSML_LAUNCH_CHECK();
    // Z = (U0+U1)(V0+V1) on the tensor cores where it pays, else the CUDA-core ring GEMM
    if (c->use_tc(M, K, N)) {
        const size_t need = tc_ring_gemm_ws_bytes(8 * (int)sizeof(T), M, K, N);
        PSML_TRY(c->ensure_ws(need));
        psml_status st = tc_dealer_gemm(8 * (int)sizeof(T), U[0], U[1], V[0], V[1], M, K, N, Z[0], Z[1], c->ws,
                                        c->ws_bytes, s);
        if (st != PSML_ERR_UNSUPPORTED) return st;
    }
    PSML_TRY(c->ensure_ws(sizeof(T) * M * N));
    T *part = (T *)c->ws;
    DealerOps<T> ops;
    ops.U0 = (const T *)U[0]; ops.U1 = (const T *)U[1]; ops.V0 = (const T *)V[0]; ops.V1 = (const T *)V[1];
    ops.Z0 = (const T *)Z[0]; ops.Z1 = (T *)Z[1];
    ops.M = M; ops.N = N; ops.Kext = K;
    return launch_ring_gemm<T, DealerOps<T>>(ops, part, M * N, s, c->sm_count);
}

psml_status psml_triplet_gen(psml_ctx ctx, uint64_t seed, uint64_t call_id, int64_t M, int64_t K, int64_t N,
                             void *const U[2], void *const V[2], void *const Z[2], psml_stream stream) {
    PSML_CTX_OPTS(ctx);
    if (!ctx) return fail(PSML_ERR_INVALID, "ctx is null");
    Ctx *c = reinterpret_cast<Ctx *>(ctx);
    if (M <= 0 || K <= 0 || N <= 0) return fail(PSML_ERR_SHAPE, "M, K, N must be positive");
    if (!U || !V || !Z) return fail(PSML_ERR_INVALID, "null pair array");
    PSML_TRY(check_ptrs({U[0], U[1], V[0], V[1], Z[0], Z[1]}));
    cudaStream_t s = (cudaStream_t)stream;
    if (c->ring.l == 64) return triplet_gen_t<uint64_t>(c, seed, call_id, 0, M, K, N, U, V, Z, s);
    return triplet_gen_t<uint32_t>(c, seed, call_id, 0, M, K, N, U, V, Z, s);
}

psml_status psml_triplet_gen_rows(psml_ctx ctx, uint64_t seed, uint64_t call_id, int64_t M_total, int64_t row0,
                                  int64_t M, int64_t K, int64_t N, void *const U[2], void *const V[2],
                                  void *const Z[2], psml_stream stream) {
    PSML_CTX_OPTS(ctx);
    if (!ctx) return fail(PSML_ERR_INVALID, "ctx is null");
    Ctx *c = reinterpret_cast<Ctx *>(ctx);
    if (M <= 0 || K <= 0 || N <= 0 || row0 < 0 || row0 + M > M_total)
        return fail(PSML_ERR_SHAPE, "rows [row0, row0 + M) must lie in [0, M_total); M, K, N > 0");
    if (!U || !V || !Z) return fail(PSML_ERR_INVALID, "null pair array");
    PSML_TRY(check_ptrs({U[0], U[1], V[0], V[1], Z[0], Z[1]}));
    cudaStream_t s = (cudaStream_t)stream;
    if (c->ring.l == 64) return triplet_gen_t<uint64_t>(c, seed, call_id, row0, M, K, N, U, V, Z, s);
    return triplet_gen_t<uint32_t>(c, seed, call_id, row0, M, K, N, U, V, Z, s);
}

psml_status psml_hadamard_triplet_gen(psml_ring ring, uint64_t seed, uint64_t call_id, int64_t n, void *const U[2],
                                      void *const V[2], void *const Z[2], psml_stream stream) {
    PSML_TRY(check_ring(ring));
    if (n < 0) return fail(PSML_ERR_SHAPE, "n < 0");
    if (n == 0) return PSML_OK;
    if (!U || !V || !Z) return fail(PSML_ERR_INVALID, "null pair array");
    PSML_TRY(check_ptrs({U[0], U[1], V[0], V[1], Z[0], Z[1]}));
    cudaStream_t s = (cudaStream_t)stream;
    if (ring.l == 64)
        return hadamard_triplet_launch<uint64_t>(dealer_seeds(seed), call_id, n, U, V, Z, s);
    return hadamard_triplet_launch<uint32_t>(dealer_seeds(seed), call_id, n, U, V, Z, s);
}

int64_t psml_msb_material_words(psml_ring ring, int64_t n) {
    if (ring.l != 32 && ring.l != 64) return -1;
    return (int64_t)MSB_WORDS * n;   // reduced prefix material (R27)
}

psml_status psml_msb_dealer(psml_ring ring, uint64_t seed, uint64_t call_id, int64_t n, void *const mat[2],
                            psml_stream stream) {
    PSML_TRY(check_ring(ring));
    if (n < 0) return fail(PSML_ERR_SHAPE, "n < 0");
    if (n == 0) return PSML_OK;
    if (!mat) return fail(PSML_ERR_INVALID, "null pair array");
    PSML_TRY(check_ptrs({mat[0], mat[1]}));
    cudaStream_t s = (cudaStream_t)stream;
    if (ring.l == 64) return msb_dealer_launch<uint64_t>(dealer_seeds(seed), call_id, n, mat, s);
    return msb_dealer_launch<uint32_t>(dealer_seeds(seed), call_id, n, mat, s);
}

// ------------------------------------------------------------------------------------------------
// server side
// ------------------------------------------------------------------------------------------------
// Config 1 (one linear-regression minibatch, A M x K . B K x 1) in ONE launch: a CTA per output
// row, both parties; its 8 warps split K.  Each thread re-derives the opened F = (B_0 - V_0) +
// (B_1 - V_1) of its K columns (K words, L2-resident) and the opened row E_m = (A_0 - U_0) +
// (A_1 - U_1) (Eqs. 4-5), accumulates p E_m.F + E_m.V_p + U_p[m].F (BJ form, the Eq. 8
// K-concatenation), and the CTA adds Z_p[m] and truncates -- the mask, open and GEMV rounds of the
// co-resident pair fused.
template <typename T>
__global__ void __launch_bounds__(256) beaver_gemv_kernel(CPair<T> A, CPair<T> B, CPair<T> U, CPair<T> V, CPair<T> Z,
                                                          int64_t M, int64_t K, int trunc, Pair<T> C) {
    __shared__ T red[2][8];
    const int64_t row = blockIdx.x;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    T acc0 = 0, acc1 = 0;
    const T *a0 = A.p[0] + row * K, *a1 = A.p[1] + row * K, *u0 = U.p[0] + row * K, *u1 = U.p[1] + row * K;
#pragma unroll 2
    for (int64_t k = tid; k < K; k += 256) {
        const T f = (B.p[0][k] - V.p[0][k]) + (B.p[1][k] - V.p[1][k]);
        const T uu0 = __ldcs(u0 + k), uu1 = __ldcs(u1 + k);
        const T e = (__ldcs(a0 + k) - uu0) + (__ldcs(a1 + k) - uu1);
        acc0 += e * V.p[0][k] + uu0 * f;
        acc1 += e * f + e * V.p[1][k] + uu1 * f;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        acc0 += __shfl_xor_sync(0xffffffffu, acc0, o);
        acc1 += __shfl_xor_sync(0xffffffffu, acc1, o);
    }
    if (lane == 0) { red[0][warp] = acc0; red[1][warp] = acc1; }
    __syncthreads();
    if (tid < 2) {
        T acc = 0;
#pragma unroll
        for (int w = 0; w < 8; ++w) acc += red[tid][w];
        C.p[tid][row] = trunc_share<T>(acc + Z.p[tid][row], tid, trunc);
    }
}

template <typename T>
static psml_status secure_matmul_t(Ctx *c, const void *const A[2], const void *const B[2], const void *const U[2],
                                   const void *const V[2], const void *const Z[2], int64_t M, int64_t K, int64_t N,
                                   int32_t flags, int32_t trunc, void *const C[2], const psml_trace *tr,
                                   cudaStream_t s) {
    const T *a[2] = {(const T *)A[0], (const T *)A[1]}, *b[2] = {(const T *)B[0], (const T *)B[1]};
    const T *u[2] = {(const T *)U[0], (const T *)U[1]}, *v[2] = {(const T *)V[0], (const T *)V[1]};
    const T *z[2] = {(const T *)Z[0], (const T *)Z[1]};
    T *cc[2] = {(T *)C[0], (T *)C[1]};
    if (!tr && !(flags & PSML_PAPER_FORM) && c->use_tc(M, 2 * K, N)) {
        psml_status st = tc_beaver_matmul<T>(c, a, b, u, v, z, M, K, N, flags, trunc, cc, s);
        if (st != PSML_ERR_UNSUPPORTED) return st;
    }
    if (!tr && flags == 0 && N == 1 && K <= 65536) {   // config 1: one fused launch
        ProfScope prof(PROF_GEMM, s, (double)M * 2 * K * 2);
        beaver_gemv_kernel<T><<<(unsigned)M, 256, 0, s>>>(
            CPair<T>{{a[0], a[1]}}, CPair<T>{{b[0], b[1]}}, CPair<T>{{u[0], u[1]}}, CPair<T>{{v[0], v[1]}},
            CPair<T>{{z[0], z[1]}}, M, K, trunc, Pair<T>{{cc[0], cc[1]}});
        PSML_LAUNCH_CHECK();
        return PSML_OK;
    }
    const int64_t words = beaver_ws_words<T>(M, K, N);
    PSML_TRY(c->ensure_ws(sizeof(T) * words));
    T *ws = (T *)c->ws;
    T *tE[2] = {tr ? (T *)tr->E[0] : nullptr, tr ? (T *)tr->E[1] : nullptr};
    T *tF[2] = {tr ? (T *)tr->F[0] : nullptr, tr ? (T *)tr->F[1] : nullptr};
    PSML_TRY(beaver_matmul<T>(a, b, u, v, z, M, K, N, flags, trunc, cc, ws, words, s, c->sm_count, tE, tF));
    if (tr) PSML_TRY(trace_opened<T>(c, M, K, N, tr, s));
    return PSML_OK;
}

psml_status psml_secure_matmul(psml_ctx ctx, const void *const A[2], const void *const B[2], const void *const U[2],
                               const void *const V[2], const void *const Z[2], int64_t M, int64_t K, int64_t N,
                               int32_t flags, int32_t trunc_bits, void *const C[2], const psml_trace *trace,
                               psml_stream stream) {
    PSML_CTX_OPTS(ctx);
    if (!ctx) return fail(PSML_ERR_INVALID, "ctx is null");
    Ctx *c = reinterpret_cast<Ctx *>(ctx);
    if (M <= 0 || K <= 0 || N <= 0) return fail(PSML_ERR_SHAPE, "M, K, N must be positive");
    if (trunc_bits < 0 || trunc_bits >= c->ring.l) return fail(PSML_ERR_SHAPE, "trunc_bits must be in [0, l)");
    if (flags & ~(PSML_TRANS_A | PSML_TRANS_B | PSML_PAPER_FORM)) return fail(PSML_ERR_INVALID, "unknown flag bits");
    if (!A || !B || !U || !V || !Z || !C) return fail(PSML_ERR_INVALID, "null pair array");
    PSML_TRY(check_ptrs({A[0], A[1], B[0], B[1], U[0], U[1], V[0], V[1], Z[0], Z[1], C[0], C[1]}));
    cudaStream_t s = (cudaStream_t)stream;
    if (c->ring.l == 64) return secure_matmul_t<uint64_t>(c, A, B, U, V, Z, M, K, N, flags, trunc_bits, C, trace, s);
    return secure_matmul_t<uint32_t>(c, A, B, U, V, Z, M, K, N, flags, trunc_bits, C, trace, s);
}

template <typename T>
static psml_status beaver_mask_t(const void *A, const void *B, const void *U, const void *V, int64_t M, int64_t K,
                                 int64_t N, int32_t flags, void *E, void *F, cudaStream_t s) {
    MaskJobs<T> jobs;
    jobs.j[0] = {(const T *)A, (const T *)U, (T *)E, M, K, (flags & PSML_TRANS_A) ? 1 : 0};
    jobs.j[1] = {(const T *)B, (const T *)V, (T *)F, K, N, (flags & PSML_TRANS_B) ? 1 : 0};
    jobs.count = 2;
    const int64_t maxt = std::max(((M + 31) / 32) * ((K + 31) / 32), ((K + 31) / 32) * ((N + 31) / 32));
    ProfScope prof(PROF_MASK, s, 3.0 * sizeof(T) * (M * K + K * N));
    mask_kernel<T><<<dim3((unsigned)std::min<int64_t>(maxt, 148 * 8), 1, 2), dim3(32, 8), 0, s>>>(jobs);
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

psml_status psml_beaver_mask(psml_ctx ctx, int32_t party, const void *A_i, const void *B_i, const void *U_i,
                             const void *V_i, int64_t M, int64_t K, int64_t N, int32_t flags, void *E_send,
                             void *F_send, psml_stream stream) {
    PSML_CTX_OPTS(ctx);
    if (!ctx) return fail(PSML_ERR_INVALID, "ctx is null");
    Ctx *c = reinterpret_cast<Ctx *>(ctx);
    if (party != 0 && party != 1) return fail(PSML_ERR_INVALID, "party must be 0 or 1");
    if (M <= 0 || K <= 0 || N <= 0) return fail(PSML_ERR_SHAPE, "M, K, N must be positive");
    if (flags & ~(PSML_TRANS_A | PSML_TRANS_B)) return fail(PSML_ERR_INVALID, "flags: TRANS_A / TRANS_B only");
    PSML_TRY(check_ptrs({A_i, B_i, U_i, V_i, E_send, F_send}));
    cudaStream_t s = (cudaStream_t)stream;
    if (c->ring.l == 64) return beaver_mask_t<uint64_t>(A_i, B_i, U_i, V_i, M, K, N, flags, E_send, F_send, s);
    return beaver_mask_t<uint32_t>(A_i, B_i, U_i, V_i, M, K, N, flags, E_send, F_send, s);
}

template <typename T>
static psml_status open_matmul_t(Ctx *c, int party, const void *Es, const void *Er, const void *Fs, const void *Fr,
                                 const void *U, const void *V, const void *Z, int64_t M, int64_t K, int64_t N,
                                 int trunc, void *C, cudaStream_t s) {
    if (c->use_tc(M, 2 * K, N)) {
        psml_status st = tc_open_matmul_one(c, 8 * (int)sizeof(T), party, Es, Er, Fs, Fr, U, V, Z, M, K, N, trunc, C, s);
        if (st != PSML_ERR_UNSUPPORTED) return st;
    }
    if (seg_eligible(M, K, N, 1) && simt_cl_enabled()) {   // open once, then the two-segment GEMM
        PSML_TRY(c->ensure_ws(sizeof(T) * (2 * M * K + K * N)));
        T *E = (T *)c->ws, *X = E + M * K, *F = X + M * K;
        OpenJobs<T> oj;
        oj.j[0] = {{(const T *)Es, (const T *)Er}, {nullptr, nullptr}, E, X, (const T *)U, (T)party, M, K, 0};
        oj.j[1] = {{(const T *)Fs, (const T *)Fr}, {nullptr, nullptr}, F, nullptr, nullptr, (T)0, K, N, 0};
        PSML_TRY(launch_open<T>(oj, s));
        SegArgs<T> sa{};
        sa.X[0] = X; sa.E = E; sa.F = F; sa.V[0] = (const T *)V; sa.Z[0] = (const T *)Z; sa.C[0] = (T *)C;
        sa.party[0] = party;
        sa.M = M; sa.N = N; sa.K = K; sa.trunc = trunc;
        return launch_seg_gemm<T>(sa, 1, s, c->sm_count);
    }
    PSML_TRY(c->ensure_ws(sizeof(T) * M * N));
    BeaverOps1<T> ops;
    ops.mE0 = (const T *)Es; ops.mE1 = (const T *)Er; ops.mF0 = (const T *)Fs; ops.mF1 = (const T *)Fr;
    ops.U = (const T *)U; ops.V = (const T *)V; ops.Z = (const T *)Z; ops.C = (T *)C;
    ops.M = M; ops.N = N; ops.K = K; ops.Kext = 2 * K; ops.party = party; ops.trunc = trunc;
    return launch_ring_gemm<T, BeaverOps1<T>>(ops, (T *)c->ws, M * N, s, c->sm_count);
}

psml_status psml_beaver_open_matmul(psml_ctx ctx, int32_t party, const void *E_send, const void *E_recv,
                                    const void *F_send, const void *F_recv, const void *U_i, const void *V_i,
                                    const void *Z_i, int64_t M, int64_t K, int64_t N, int32_t trunc_bits, void *C_i,
                                    psml_stream stream) {
    PSML_CTX_OPTS(ctx);
    if (!ctx) return fail(PSML_ERR_INVALID, "ctx is null");
    Ctx *c = reinterpret_cast<Ctx *>(ctx);
    if (party != 0 && party != 1) return fail(PSML_ERR_INVALID, "party must be 0 or 1");
    if (M <= 0 || K <= 0 || N <= 0) return fail(PSML_ERR_SHAPE, "M, K, N must be positive");
    if (trunc_bits < 0 || trunc_bits >= c->ring.l) return fail(PSML_ERR_SHAPE, "trunc_bits must be in [0, l)");
    PSML_TRY(check_ptrs({E_send, E_recv, F_send, F_recv, U_i, V_i, Z_i, C_i}));
    cudaStream_t s = (cudaStream_t)stream;
    if (c->ring.l == 64)
        return open_matmul_t<uint64_t>(c, party, E_send, E_recv, F_send, F_recv, U_i, V_i, Z_i, M, K, N, trunc_bits,
                                       C_i, s);
    return open_matmul_t<uint32_t>(c, party, E_send, E_recv, F_send, F_recv, U_i, V_i, Z_i, M, K, N, trunc_bits, C_i,
                                   s);
}

psml_status psml_secure_hadamard(psml_ctx ctx, const void *const A[2], const void *const B[2], const void *const U[2],
                                 const void *const V[2], const void *const Z[2], int64_t n, int32_t trunc_bits,
                                 void *const C[2], psml_stream stream) {
    PSML_CTX_OPTS(ctx);
    if (!ctx) return fail(PSML_ERR_INVALID, "ctx is null");
    Ctx *c = reinterpret_cast<Ctx *>(ctx);
    if (n < 0) return fail(PSML_ERR_SHAPE, "n < 0");
    if (trunc_bits < 0 || trunc_bits >= c->ring.l) return fail(PSML_ERR_SHAPE, "trunc_bits must be in [0, l)");
    if (n == 0) return PSML_OK;
    if (!A || !B || !U || !V || !Z || !C) return fail(PSML_ERR_INVALID, "null pair array");
    PSML_TRY(check_ptrs({A[0], A[1], B[0], B[1], U[0], U[1], V[0], V[1], Z[0], Z[1], C[0], C[1]}));
    cudaStream_t s = (cudaStream_t)stream;
    if (c->ring.l == 64) {
        PSML_TRY(c->ensure_ws(sizeof(uint64_t) * 4 * n));
        return beaver_hadamard<uint64_t>((const uint64_t *const *)A, (const uint64_t *const *)B, (const uint64_t *const *)U,
                                         (const uint64_t *const *)V, (const uint64_t *const *)Z, n, trunc_bits,
                                         (uint64_t *const *)C, (uint64_t *)c->ws, s);
    }
    PSML_TRY(c->ensure_ws(sizeof(uint32_t) * 4 * n));
    return beaver_hadamard<uint32_t>((const uint32_t *const *)A, (const uint32_t *const *)B, (const uint32_t *const *)U,
                                     (const uint32_t *const *)V, (const uint32_t *const *)Z, n, trunc_bits,
                                     (uint32_t *const *)C, (uint32_t *)c->ws, s);
}

psml_status psml_truncate(psml_ring ring, int32_t party, void *x_i, int64_t n, int32_t bits, psml_stream stream) {
    PSML_TRY(check_ring(ring));
    if (party != 0 && party != 1) return fail(PSML_ERR_INVALID, "party must be 0 or 1");
    if (n < 0 || bits < 0 || bits >= ring.l) return fail(PSML_ERR_SHAPE, "bad n or bits");
    if (n == 0 || bits == 0) return PSML_OK;
    PSML_TRY(check_ptrs({x_i}));
    cudaStream_t s = (cudaStream_t)stream;
    if (ring.l == 64) truncate_kernel<uint64_t><<<grid_for(n, 256), 256, 0, s>>>((uint64_t *)x_i, n, party, bits);
    else truncate_kernel<uint32_t><<<grid_for(n, 256), 256, 0, s>>>((uint32_t *)x_i, n, party, bits);
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

template <typename T>
static psml_status activation_t(Ctx *c, int what, const void *const x[2], int64_t n, const void *const mat[2],
                                void *const msbA[2], void *const msbB[2], const void *const U[2],
                                const void *const V[2], const void *const Z[2], void *const y[2],
                                void *const drelu[2], cudaStream_t s) {
    const int64_t nn = what == 2 ? 2 * n : n;  // Eq. 9 runs the chain on [x + 1/2 ; x - 1/2]
    PSML_TRY(c->ensure_ws(sizeof(T) * msb_ws_words<T>(nn)));
    const T half = (T)1 << (c->ring.frac_bits > 0 ? c->ring.frac_bits - 1 : 0);
    return msb_chain<T>((const T *const *)x, nn, (const T *const *)mat, what == 2 ? 1 : 0, half, what,
                        (T *const *)msbA, (T *const *)msbB, (T *const *)drelu, (const T *const *)U,
                        (const T *const *)V, (const T *const *)Z, (T *const *)y, nullptr, nullptr, (T *)c->ws, s);
}

psml_status psml_secure_msb(psml_ctx ctx, const void *const x[2], int64_t n, const void *const mat[2],
                            void *const msbA[2], void *const msbB[2], psml_stream stream) {
    PSML_CTX_OPTS(ctx);
    if (!ctx) return fail(PSML_ERR_INVALID, "ctx is null");
    Ctx *c = reinterpret_cast<Ctx *>(ctx);
    if (n < 0) return fail(PSML_ERR_SHAPE, "n < 0");
    if (n == 0) return PSML_OK;
    if (!x || !mat || !msbA) return fail(PSML_ERR_INVALID, "null pair array");
    PSML_TRY(check_ptrs({x[0], x[1], mat[0], mat[1], msbA[0], msbA[1]}));
    cudaStream_t s = (cudaStream_t)stream;
    if (c->ring.l == 64) return activation_t<uint64_t>(c, 0, x, n, mat, msbA, msbB, nullptr, nullptr, nullptr, nullptr, nullptr, s);
    return activation_t<uint32_t>(c, 0, x, n, mat, msbA, msbB, nullptr, nullptr, nullptr, nullptr, nullptr, s);
}

psml_status psml_secure_relu(psml_ctx ctx, const void *const x[2], int64_t n, const void *const mat[2],
                             const void *const U[2], const void *const V[2], const void *const Z[2], void *const y[2],
                             void *const drelu[2], psml_stream stream) {
    PSML_CTX_OPTS(ctx);
    if (!ctx) return fail(PSML_ERR_INVALID, "ctx is null");
    Ctx *c = reinterpret_cast<Ctx *>(ctx);
    if (n < 0) return fail(PSML_ERR_SHAPE, "n < 0");
    if (n == 0) return PSML_OK;
    if (!x || !mat || !U || !V || !Z || !y) return fail(PSML_ERR_INVALID, "null pair array");
    PSML_TRY(check_ptrs({x[0], x[1], mat[0], mat[1], U[0], U[1], V[0], V[1], Z[0], Z[1], y[0], y[1]}));
    cudaStream_t s = (cudaStream_t)stream;
    if (c->ring.l == 64) return activation_t<uint64_t>(c, 1, x, n, mat, nullptr, nullptr, U, V, Z, y, drelu, s);
    return activation_t<uint32_t>(c, 1, x, n, mat, nullptr, nullptr, U, V, Z, y, drelu, s);
}

psml_status psml_secure_eq9(psml_ctx ctx, const void *const x[2], int64_t n, const void *const mat[2],
                            const void *const U[2], const void *const V[2], const void *const Z[2], void *const y[2],
                            psml_stream stream) {
    if (!ctx) return fail(PSML_ERR_INVALID, "ctx is null");
    Ctx *c = reinterpret_cast<Ctx *>(ctx);
    if (n < 0) return fail(PSML_ERR_SHAPE, "n < 0");
    if (n == 0) return PSML_OK;
    if (!x || !mat || !U || !V || !Z || !y) return fail(PSML_ERR_INVALID, "null pair array");
    PSML_TRY(check_ptrs({x[0], x[1], mat[0], mat[1], U[0], U[1], V[0], V[1], Z[0], Z[1], y[0], y[1]}));
    cudaStream_t s = (cudaStream_t)stream;
    if (c->ring.l == 64) return activation_t<uint64_t>(c, 2, x, n, mat, nullptr, nullptr, U, V, Z, y, nullptr, s);
    return activation_t<uint32_t>(c, 2, x, n, mat, nullptr, nullptr, U, V, Z, y, nullptr, s);
}

// ------------------------------------------------------------------------------------------------
// one-round FSS comparison (fss.cuh, R22); Z_2^64 only
// ------------------------------------------------------------------------------------------------
int64_t psml_fss_material_words(psml_ring ring, int64_t n) {
    if (ring.l != 64 || n < 0) return -1;
    return (int64_t)FSS_WORDS * n;
}

psml_status psml_fss_dealer(psml_ring ring, uint64_t seed, uint64_t call_id, int64_t n, void *const mat[2],
                            psml_stream stream) {
    PSML_TRY(check_ring(ring));
    if (ring.l != 64) return fail(PSML_ERR_UNSUPPORTED, "the FSS comparison is built for Z_2^64");
    if (n < 0) return fail(PSML_ERR_SHAPE, "n < 0");
    if (n == 0) return PSML_OK;
    if (!mat) return fail(PSML_ERR_INVALID, "null pair array");
    PSML_TRY(check_ptrs({mat[0], mat[1]}));
    cudaStream_t s = (cudaStream_t)stream;
    ProfScope prof(PROF_DEALER, s, 2.0 * FSS_BITS * (double)n);
    return fss_dealer_launch(dealer_seeds(seed), call_id, n, (uint64_t *)mat[0], (uint64_t *)mat[1], s);
}

static psml_status fss_drelu_pair(const void *const x[2], int64_t n, const void *const mat[2], uint64_t *const d[2],
                                  uint64_t *xhat, uint64_t *ws, cudaStream_t s) {
    return fss_drelu_launch(CPair<uint64_t>{{(const uint64_t *)x[0], (const uint64_t *)x[1]}}, n,
                            CPair<uint64_t>{{(const uint64_t *)mat[0], (const uint64_t *)mat[1]}},
                            Pair<uint64_t>{{d[0], d[1]}}, xhat, ws, s);
}

psml_status psml_secure_drelu_fss(psml_ctx ctx, const void *const x[2], int64_t n, const void *const mat[2],
                                  void *const drelu[2], void *xhat_trace, psml_stream stream) {
    PSML_CTX_OPTS(ctx);
    if (!ctx) return fail(PSML_ERR_INVALID, "ctx is null");
    Ctx *c = reinterpret_cast<Ctx *>(ctx);
    if (c->ring.l != 64) return fail(PSML_ERR_UNSUPPORTED, "the FSS comparison is built for Z_2^64");
    if (n < 0) return fail(PSML_ERR_SHAPE, "n < 0");
    if (n == 0) return PSML_OK;
    if (!x || !mat || !drelu) return fail(PSML_ERR_INVALID, "null pair array");
    PSML_TRY(check_ptrs({x[0], x[1], mat[0], mat[1], drelu[0], drelu[1], xhat_trace}));
    PSML_TRY(c->ensure_ws(sizeof(uint64_t) * 2 * n));
    uint64_t *d[2] = {(uint64_t *)drelu[0], (uint64_t *)drelu[1]};
    return fss_drelu_pair(x, n, mat, d, (uint64_t *)xhat_trace, (uint64_t *)c->ws, (cudaStream_t)stream);
}

psml_status psml_secure_relu_fss(psml_ctx ctx, const void *const x[2], int64_t n, const void *const mat[2],
                                 const void *const U[2], const void *const V[2], const void *const Z[2],
                                 void *const y[2], void *const drelu[2], psml_stream stream) {
    PSML_CTX_OPTS(ctx);
    if (!ctx) return fail(PSML_ERR_INVALID, "ctx is null");
    Ctx *c = reinterpret_cast<Ctx *>(ctx);
    if (c->ring.l != 64) return fail(PSML_ERR_UNSUPPORTED, "the FSS comparison is built for Z_2^64");
    if (n < 0) return fail(PSML_ERR_SHAPE, "n < 0");
    if (n == 0) return PSML_OK;
    if (!x || !mat || !U || !V || !Z || !y) return fail(PSML_ERR_INVALID, "null pair array");
    PSML_TRY(check_ptrs({x[0], x[1], mat[0], mat[1], U[0], U[1], V[0], V[1], Z[0], Z[1], y[0], y[1]}));
    if (drelu) PSML_TRY(check_ptrs({drelu[0], drelu[1]}));
    PSML_TRY(c->ensure_ws(sizeof(uint64_t) * 8 * n));
    uint64_t *ws = (uint64_t *)c->ws;
    uint64_t *d[2] = {drelu ? (uint64_t *)drelu[0] : ws + 2 * n, drelu ? (uint64_t *)drelu[1] : ws + 3 * n};
    cudaStream_t s = (cudaStream_t)stream;
    PSML_TRY(fss_drelu_pair(x, n, mat, d, nullptr, ws, s));
    const uint64_t *A[2] = {(const uint64_t *)x[0], (const uint64_t *)x[1]};
    const uint64_t *Bd[2] = {d[0], d[1]};
    return beaver_hadamard<uint64_t>(A, Bd, (const uint64_t *const *)U, (const uint64_t *const *)V,
                                     (const uint64_t *const *)Z, n, 0, (uint64_t *const *)y, ws + 4 * n, s);
}

// split deployment: party `party`'s round-1 message and its evaluation after the exchange
psml_status psml_fss_mask(psml_ctx ctx, int32_t party, const void *x_i, int64_t n, const void *mat_i, void *msg,
                          psml_stream stream) {
    PSML_CTX_OPTS(ctx);
    if (!ctx) return fail(PSML_ERR_INVALID, "ctx is null");
    if (party != 0 && party != 1) return fail(PSML_ERR_INVALID, "party must be 0 or 1");
    if (reinterpret_cast<Ctx *>(ctx)->ring.l != 64) return fail(PSML_ERR_UNSUPPORTED, "Z_2^64 only");
    if (n < 0) return fail(PSML_ERR_SHAPE, "n < 0");
    if (n == 0) return PSML_OK;
    PSML_TRY(check_ptrs({x_i, mat_i, msg}));
    CPair<uint64_t> xx{{nullptr, nullptr}}, mm{{nullptr, nullptr}};
    Pair<uint64_t> out{{nullptr, nullptr}};
    xx.p[party] = (const uint64_t *)x_i; mm.p[party] = (const uint64_t *)mat_i; out.p[party] = (uint64_t *)msg;
    fss_mask_kernel<<<ew_grid(n), EW_THREADS, 0, (cudaStream_t)stream>>>(xx, mm, n, out, party);
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

psml_status psml_fss_open_drelu(psml_ctx ctx, int32_t party, const void *msg_send, const void *msg_recv, int64_t n,
                                const void *mat_i, void *drelu_i, psml_stream stream) {
    PSML_CTX_OPTS(ctx);
    if (!ctx) return fail(PSML_ERR_INVALID, "ctx is null");
    if (party != 0 && party != 1) return fail(PSML_ERR_INVALID, "party must be 0 or 1");
    if (reinterpret_cast<Ctx *>(ctx)->ring.l != 64) return fail(PSML_ERR_UNSUPPORTED, "Z_2^64 only");
    if (n < 0) return fail(PSML_ERR_SHAPE, "n < 0");
    if (n == 0) return PSML_OK;
    PSML_TRY(check_ptrs({msg_send, msg_recv, mat_i, drelu_i}));
    CPair<uint64_t> msg{{nullptr, nullptr}}, mm{{nullptr, nullptr}};
    msg.p[party] = (const uint64_t *)msg_send;
    msg.p[1 - party] = (const uint64_t *)msg_recv;
    mm.p[party] = (const uint64_t *)mat_i;
    Pair<uint64_t> d{{nullptr, nullptr}};
    d.p[party] = (uint64_t *)drelu_i;
    fss_eval_kernel<<<grid_for(n, 128, 148 * 16), 128, 0, (cudaStream_t)stream>>>(msg, mm, n, d, nullptr, party);
    PSML_LAUNCH_CHECK();
    return PSML_OK;
}

template <typename T>
static psml_status ring_gemm_t(Ctx *c, const void *A, const void *B, int64_t M, int64_t K, int64_t N, void *C,
                               cudaStream_t s) {
    if (c->use_tc(M, K, N) && tc_seg_small(8 * (int)sizeof(T), M, K, N, 1, c->sm_count))   // one launch
        return tc_seg_plain<T>((const T *)A, (const T *)B, M, K, N, (T *)C, s, c->sm_count);
    if (c->use_tc(M, K, N)) {
        size_t need = tc_ring_gemm_ws_bytes(8 * (int)sizeof(T), M, K, N);
        PSML_TRY(c->ensure_ws(need));
        psml_status st = tc_ring_gemm_plain(8 * (int)sizeof(T), A, B, M, K, N, C, c->ws, c->ws_bytes, s);
        if (st != PSML_ERR_UNSUPPORTED) return st;
    }
    PSML_TRY(c->ensure_ws(sizeof(T) * M * N));
    PlainOps<T> ops;
    ops.A = (const T *)A; ops.B = (const T *)B; ops.C = (T *)C;
    ops.M = M; ops.N = N; ops.Kext = K;
    return launch_ring_gemm<T, PlainOps<T>>(ops, (T *)c->ws, M * N, s, c->sm_count);
}

psml_status psml_ring_gemm(psml_ctx ctx, const void *A, const void *B, int64_t M, int64_t K, int64_t N, void *C,
                           psml_stream stream) {
    PSML_CTX_OPTS(ctx);
    if (!ctx) return fail(PSML_ERR_INVALID, "ctx is null");
    Ctx *c = reinterpret_cast<Ctx *>(ctx);
    if (M <= 0 || K <= 0 || N <= 0) return fail(PSML_ERR_SHAPE, "M, K, N must be positive");
    PSML_TRY(check_ptrs({A, B, C}));
    cudaStream_t s = (cudaStream_t)stream;
    if (c->ring.l == 64) return ring_gemm_t<uint64_t>(c, A, B, M, K, N, C, s);
    return ring_gemm_t<uint32_t>(c, A, B, M, K, N, C, s);
}

