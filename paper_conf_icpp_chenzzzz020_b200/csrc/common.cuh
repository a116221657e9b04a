// common.cuh -- shared device helpers of libpsml (CUDA path).  Independent of oracle/.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>
#include <string>

#pragma GCC visibility push(default)
#include "../../include/psml.h"
#pragma GCC visibility pop

namespace psml {

// ---------------------------------------------------------------------------------------------
// error plumbing (no exceptions cross the ABI)
// ---------------------------------------------------------------------------------------------
void set_error(const std::string &msg);
psml_status fail(psml_status st, const std::string &msg);
extern std::atomic<uint64_t> g_launches;

#define PSML_CUDA_TRY(expr)                                                                     \
    do {                                                                                        \
        cudaError_t _e = (expr);                                                                \
        if (_e != cudaSuccess)                                                                  \
            return ::psml::fail(PSML_ERR_CUDA, std::string(#expr) + ": " + cudaGetErrorString(_e)); \
    } while (0)

#define PSML_LAUNCH_CHECK()                                                                     \
    do {                                                                                        \
        ::psml::g_launches.fetch_add(1, std::memory_order_relaxed);                             \
        cudaError_t _e = cudaGetLastError();                                                    \
        if (_e != cudaSuccess)                                                                  \
            return ::psml::fail(PSML_ERR_CUDA, std::string("kernel launch: ") + cudaGetErrorString(_e)); \
    } while (0)

// ---------------------------------------------------------------------------------------------
// kernel-class profiling (psml_prof_enable / psml_prof_read): CUDA events around launches
// ---------------------------------------------------------------------------------------------
enum ProfClass { PROF_GEMM = 0, PROF_TC = 1, PROF_MSB = 2, PROF_HAD = 3, PROF_DEALER = 4, PROF_MASK = 5 };
extern std::atomic<int> g_prof_cls;
void prof_record(cudaEvent_t a, cudaEvent_t b, double work);
cudaEvent_t prof_event();

struct ProfScope {
    bool on = false;
    cudaEvent_t a = nullptr;
    cudaStream_t s = nullptr;
    double work = 0;
    ProfScope(int cls, cudaStream_t st, double w) {
        if (g_prof_cls.load(std::memory_order_relaxed) == cls) {
            on = true; s = st; work = w;
            a = prof_event();
            cudaEventRecord(a, s);
        }
    }
    ~ProfScope() {
        if (on) {
            cudaEvent_t b = prof_event();
            cudaEventRecord(b, s);
            prof_record(a, b, work);
        }
    }
};

// Programmatic dependent launch trigger: lets a dependent kernel launched with
// cudaLaunchAttributeProgrammaticStreamSerialization start its prologue now (it still waits,
// with griddepcontrol.wait, for this grid's completion before reading its outputs).
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
// Wait for the predecessor grid's completion and memory flush (a no-op without a programmatic
// dependency).  Every PDL-launched kernel calls it before touching its predecessor's outputs.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
bool pdl_enabled();   // PSML_PDL=0 disables programmatic dependent launch

// <<<grid, block, 0, s>>> with programmatic stream serialization (PDL): the kernel may be
// scheduled while its predecessor drains; it must pdl_wait() before reading the predecessor's data.
template <typename... KArgs, typename... Args>
cudaError_t launch_pdl(void (*k)(KArgs...), dim3 grid, dim3 block, cudaStream_t s, Args... args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = pdl_enabled() ? 1 : 0;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, k, args...);
}

#define PSML_TRY(expr)                          \
    do {                                        \
        psml_status _s = (expr);                \
        if (_s != PSML_OK) return _s;           \
    } while (0)

// ---------------------------------------------------------------------------------------------
// role tags (4 bytes, little endian) -- DESIGN.md R1/R4/R9
// ---------------------------------------------------------------------------------------------
constexpr uint32_t tag4(char a, char b, uint32_t c = 0, uint32_t d = 0) {
    return (uint32_t)(uint8_t)a | ((uint32_t)(uint8_t)b << 8) | ((c & 0xFFu) << 16) | ((d & 0xFFu) << 24);
}
constexpr uint32_t TAG_SH = tag4('S', 'H');
constexpr uint32_t TAG_U0 = tag4('U', '0'), TAG_U1 = tag4('U', '1');
constexpr uint32_t TAG_V0 = tag4('V', '0'), TAG_V1 = tag4('V', '1');
constexpr uint32_t TAG_Z0 = tag4('Z', '0');
constexpr uint32_t TAG_R0 = tag4('R', '0'), TAG_R1 = tag4('R', '1'), TAG_RA = tag4('R', 'A');

// ---------------------------------------------------------------------------------------------
// ChaCha20 block function (RFC 8439 Sec. 2.3), fully unrolled in registers
// ---------------------------------------------------------------------------------------------
__device__ __forceinline__ uint32_t rotl(uint32_t v, int c) { return __funnelshift_l(v, v, c); }

#define PSML_QR(a, b, c, d)              \
    a += b; d ^= a; d = rotl(d, 16);     \
    c += d; b ^= c; b = rotl(b, 12);     \
    a += b; d ^= a; d = rotl(d, 8);      \
    c += d; b ^= c; b = rotl(b, 7);

struct PrgKey {
    uint32_t k0, k1;         // seed words (rest of the 256-bit key is zero)
    uint32_t n0, n1, n2;     // nonce = tag || call_id
    const uint32_t *step;    // optional: device word overriding call-id bits 55:24 (CUDA graphs)
};

__host__ __device__ inline PrgKey make_key(uint64_t seed, uint32_t tag, uint64_t call_id,
                                           const uint32_t *step = nullptr) {
    PrgKey k;
    k.k0 = (uint32_t)seed; k.k1 = (uint32_t)(seed >> 32);
    k.n0 = tag; k.n1 = (uint32_t)call_id; k.n2 = (uint32_t)(call_id >> 32);
    k.step = step;
    return k;
}

// The options of the context the current ABI call runs on (psml_options; a thread-local pointer
// set for the duration of the call -- contexts are per host thread, include/psml.h).
const psml_options &cur_opts();
// A launch-completion event for the next tcgen05 product launch (psml_options.deal_on_launch:
// the pipelined graph's dealer fork edge); take_launch_event returns and clears it.
void arm_launch_event(cudaEvent_t e);
cudaEvent_t take_launch_event();
struct OptScope {
    const psml_options *prev;
    explicit OptScope(const psml_options *o);
    ~OptScope();
};

// Dealer key separation (R23): each material stream is keyed by the seed of the party
// that can produce it alone -- s_0 for U0 V0 Z0 a0 b0 c0 R0 RA F0 FS K0, s_1 for U1 V1 a1 b1 R1 K1 --
// or by the dealer seed (the FSS input mask "FR").  s_i = PRG(dealer seed, "KD", i)[0].  A party that
// deals for itself alone holds only its s_i (the other entries are 0 and their streams are junk,
// overwritten by the dealer's bundle of derived words).
struct DealSeeds {
    uint64_t d, s0, s1;
};
__host__ __device__ inline uint64_t seed_for(const DealSeeds &S, uint32_t tag) {
    const uint32_t b0 = tag & 0xFF, b1 = (tag >> 8) & 0xFF;
    if (b1 == '1') return S.s1;
    if (b1 == '0' || (b0 == 'R' && b1 == 'A') || (b0 == 'F' && b1 == 'S')) return S.s0;
    return S.d;
}
__host__ __device__ inline PrgKey dkey(const DealSeeds &S, uint32_t tag, uint64_t call_id,
                                       const uint32_t *step = nullptr) {
    return make_key(seed_for(S, tag), tag, call_id, step);
}
// Host: the seeds of a full dealer (engine.cu).
DealSeeds dealer_seeds(uint64_t dealer_seed);

// Resolve the step field from device memory (call id = pair|step|layer|op|slot, R11),
// so a captured graph replays with a new step number without re-instantiation.
__device__ __forceinline__ PrgKey live_key(PrgKey k) {
    if (k.step) {
        const uint32_t st = *k.step;
        k.n1 = (k.n1 & 0x00FFFFFFu) | (st << 24);
        k.n2 = (k.n2 & 0xFF000000u) | (st >> 8);
    }
    return k;
}

__device__ __forceinline__ void chacha20_block(const PrgKey &key, uint32_t counter, uint32_t out[16]) {
    uint32_t x0 = 0x61707865u, x1 = 0x3320646eu, x2 = 0x79622d32u, x3 = 0x6b206574u;
    uint32_t x4 = key.k0, x5 = key.k1, x6 = 0, x7 = 0, x8 = 0, x9 = 0, x10 = 0, x11 = 0;
    uint32_t x12 = counter, x13 = key.n0, x14 = key.n1, x15 = key.n2;
#pragma unroll
    for (int r = 0; r < 10; ++r) {
        PSML_QR(x0, x4, x8, x12); PSML_QR(x1, x5, x9, x13);
        PSML_QR(x2, x6, x10, x14); PSML_QR(x3, x7, x11, x15);
        PSML_QR(x0, x5, x10, x15); PSML_QR(x1, x6, x11, x12);
        PSML_QR(x2, x7, x8, x13); PSML_QR(x3, x4, x9, x14);
    }
    out[0] = x0 + 0x61707865u; out[1] = x1 + 0x3320646eu; out[2] = x2 + 0x79622d32u;
    out[3] = x3 + 0x6b206574u; out[4] = x4 + key.k0; out[5] = x5 + key.k1; out[6] = x6;
    out[7] = x7; out[8] = x8; out[9] = x9; out[10] = x10; out[11] = x11; out[12] = x12 + counter;
    out[13] = x13 + key.n0; out[14] = x14 + key.n1; out[15] = x15 + key.n2;
}

// Single element e of a stream (used where elements are scattered: epilogues, im2col).
template <typename T>
__device__ __forceinline__ T prg_elem(const PrgKey &key, uint64_t e) {
    uint32_t blk[16];
    if (sizeof(T) == 8) {
        chacha20_block(key, (uint32_t)(e >> 3), blk);
        int j = (int)(e & 7);
        uint32_t lo = 0, hi = 0;
#pragma unroll
        for (int t = 0; t < 8; ++t)
            if (t == j) { lo = blk[2 * t]; hi = blk[2 * t + 1]; }
        return (T)(((uint64_t)hi << 32) | lo);
    } else {
        chacha20_block(key, (uint32_t)(e >> 4), blk);
        int j = (int)(e & 15);
        uint32_t v = 0;
#pragma unroll
        for (int t = 0; t < 16; ++t)
            if (t == j) v = blk[t];
        return (T)v;
    }
}

// Elements per ChaCha20 block for word type T.
template <typename T> struct PerBlock { static constexpr int value = 64 / sizeof(T); };

// Truncation (SecureML local, R7) on l-bit words stored in T (l = 8 sizeof(T)).
template <typename T>
__device__ __forceinline__ T trunc_share(T v, int party, int d) {
    if (d <= 0) return v;
    return party == 0 ? (T)(v >> d) : (T)((T)0 - (T)(((T)0 - v) >> d));
}

__host__ __device__ inline int ilog2_int(int l) { int L = 0; while ((1 << L) < l) ++L; return L; }

inline int grid_for(int64_t n, int threads, int max_blocks = 148 * 16) {
    int64_t b = (n + threads - 1) / threads;
    if (b < 1) b = 1;
    if (b > max_blocks) b = max_blocks;
    return (int)b;
}

inline bool aligned16(const void *p) { return p == nullptr || (((uintptr_t)p) & 15u) == 0; }

}  // namespace psml
