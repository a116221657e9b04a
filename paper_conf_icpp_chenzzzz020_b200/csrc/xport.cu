// xport.cu -- transports of the split deployment (include/psml.h "Split deployment").
//
// PAPER.md Fig. 1b (L55-L61) puts the two servers on different machines and L65 has them
// "compute E and F via communication": every opening is one symmetric exchange of the parties'
// masked messages (R5).  Two transports implement that exchange:
//   NCCL      a library-owned 2-rank communicator per party pair; one exchange = one grouped
//             ncclSend/ncclRecv per buffer on the step's stream (stream-ordered, NVLink P2P
//             between GPUs, no host synchronisation);
//   peer      peer memory (the default): each party owns a double-buffered mailbox in its HBM
//             that the peer maps (CUDA IPC across processes -- NVLink P2P between GPUs, the same
//             HBM on one GPU -- or the raw pointer inside one process).  One exchange = ONE
//             kernel on the step's stream: put my messages into the peer's mailbox with plain
//             stores, signal it with a system-scope release, wait for the peer's signal, copy my
//             mailbox out, acknowledge.  No host synchronisation, graph-capturable (sequence
//             numbers live in device memory), works on one GPU with two processes.
//   callback  a host function supplied by the caller (host-staged gloo).
#include <nccl.h>
#include <unistd.h>

#include <algorithm>
#include <cstring>
#include <string>
#include <vector>

#include "engine.h"

// flag words of a peer mailbox (each on its own 128-byte line); then the fused kernels' window
// flags (psml::PeerWindow: an epoch counter, a done counter and one flag per CTA)
enum { XF_ARRIVED = 0, XF_CONSUMED = 16, XF_SEQ = 32, XF_CNT1 = 48, XF_CNT2 = 64,
       XF_WORDS = psml::PW_FLAG_BASE + psml::PW_MAX_CTAS * psml::PW_FLAG_STRIDE };

struct psml_xport_s {
    int kind = 0;                 // 0 NCCL, 1 callback, 2 peer memory
    ncclComm_t comm = nullptr;
    int rank = 0;
    psml_exchange_fn fn = nullptr;
    void *user = nullptr;
    int64_t bytes_sent = 0, exchanges = 0;
    // peer memory
    int device = -1;
    int64_t cap = 0;              // bytes per mailbox slot
    uint8_t *my_mb = nullptr;     // 2 * cap bytes, written by the peer
    uint64_t *my_flags = nullptr; // XF_WORDS words, written by the peer (and my own counters)
    uint8_t *peer_mb = nullptr;   // the peer's mailbox (mapped)
    uint64_t *peer_flags = nullptr;
    bool peer_ipc = false;        // mapped with cudaIpcOpenMemHandle (unmap on destroy)
};

namespace psml {

static psml_status nccl_fail(ncclResult_t r, const char *what) {
    return fail(PSML_ERR_NCCL, std::string(what) + ": " + ncclGetErrorString(r));
}

}  // namespace psml

using namespace psml;

psml_status psml_nccl_unique_id(uint8_t uid[128]) {
    if (!uid) return fail(PSML_ERR_INVALID, "uid is null");
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId is 128 bytes");
    ncclUniqueId id;
    ncclResult_t r = ncclGetUniqueId(&id);
    if (r != ncclSuccess) return nccl_fail(r, "ncclGetUniqueId");
    std::memcpy(uid, &id, sizeof(id));
    return PSML_OK;
}

psml_status psml_xport_nccl_create(const uint8_t uid[128], int32_t rank, psml_xport *out) {
    if (!uid || !out) return fail(PSML_ERR_INVALID, "null argument");
    if (rank != 0 && rank != 1) return fail(PSML_ERR_INVALID, "rank (party) must be 0 or 1");
    ncclUniqueId id;
    std::memcpy(&id, uid, sizeof(id));
    ncclComm_t comm = nullptr;
    ncclResult_t r = ncclCommInitRank(&comm, 2, id, rank);
    if (r != ncclSuccess) return nccl_fail(r, "ncclCommInitRank");
    auto *x = new psml_xport_s;
    x->kind = 0;
    x->comm = comm;
    x->rank = rank;
    *out = x;
    return PSML_OK;
}

psml_status psml_xport_callback_create(psml_exchange_fn fn, void *user, psml_xport *out) {
    if (!fn || !out) return fail(PSML_ERR_INVALID, "null argument");
    auto *x = new psml_xport_s;
    x->kind = 1;
    x->fn = fn;
    x->user = user;
    *out = x;
    return PSML_OK;
}

// ------------------------------------------------------------------------------------------------
// peer-memory transport
// ------------------------------------------------------------------------------------------------
namespace psml {

struct PeerHandle {             // the PSML_PEER_HANDLE_BYTES blob shipped to the peer
    uint32_t magic, version;
    int64_t pid;
    int32_t device, party;
    uint64_t raw_mb, raw_flags;  // valid inside the creating process only
    int64_t cap;
    cudaIpcMemHandle_t mb, flags;
};
static_assert(sizeof(PeerHandle) <= PSML_PEER_HANDLE_BYTES, "peer handle blob too small");
static constexpr uint32_t PEER_MAGIC = 0x50534D58;   // "PSMX"

constexpr int XMAX = 8;
struct XPiece {
    const uint8_t *src;
    uint8_t *dst;
    int64_t bytes, off;   // off: byte offset inside the mailbox slot (16-byte aligned)
};
struct XArgs {
    XPiece p[XMAX];
    int n;
    uint8_t *peer_mb;
    const uint8_t *my_mb;
    int64_t cap;
    uint64_t *my_flags, *peer_flags;
};

__device__ __forceinline__ uint64_t ld_acquire_sys(const uint64_t *p) {
    uint64_t v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_sys(uint64_t *p, uint64_t v) {
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t gtimer() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
// Spin until *p >= want.  A peer that never answers (crashed process, mismatched call sequence)
// must not hang the GPU: after 60 s the kernel traps, which fails the step with a CUDA error.
__device__ __forceinline__ void spin_until(const uint64_t *p, uint64_t want) {
    const uint64_t t0 = gtimer();
    while (ld_acquire_sys(p) < want) {
        __nanosleep(128);
        if (gtimer() - t0 > 60ull * 1000000000ull) __trap();
    }
}

__device__ __forceinline__ void copy_bytes(uint8_t *dst, const uint8_t *src, int64_t bytes, int64_t tid, int64_t nth) {
    const uintptr_t al = ((uintptr_t)dst) | ((uintptr_t)src);
    int64_t done = 0;
    if ((al & 15) == 0) {
        const int64_t nv = bytes >> 4;
        const int4 *s4 = reinterpret_cast<const int4 *>(src);
        int4 *d4 = reinterpret_cast<int4 *>(dst);
        for (int64_t i = tid; i < nv; i += nth) d4[i] = __ldcs(s4 + i);
        done = nv << 4;
    } else if ((al & 7) == 0) {
        const int64_t nv = bytes >> 3;
        const uint64_t *s8 = reinterpret_cast<const uint64_t *>(src);
        uint64_t *d8 = reinterpret_cast<uint64_t *>(dst);
        for (int64_t i = tid; i < nv; i += nth) d8[i] = __ldcs(s8 + i);
        done = nv << 3;
    }
    for (int64_t i = done + tid; i < bytes; i += nth) dst[i] = src[i];
}

// One symmetric exchange: put -> signal -> wait -> copy out -> acknowledge (see the file header).
// Sequence s = flags[SEQ] + 1 uses mailbox slot s & 1; the put of s waits until the peer has
// consumed s - 2 from the same slot.  The grid must be co-resident-able (<= one CTA per SM).
__global__ void __launch_bounds__(512) xport_peer_kernel(const XArgs a) {
    __shared__ uint64_t s_seq;
    if (threadIdx.x == 0) s_seq = *(volatile uint64_t *)(a.my_flags + XF_SEQ) + 1;
    __syncthreads();
    const uint64_t s = s_seq;
    const int64_t slot = (int64_t)(s & 1) * a.cap;
    if (threadIdx.x == 0 && s > 2) spin_until(a.my_flags + XF_CONSUMED, s - 2);
    __syncthreads();
    const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x, nth = (int64_t)gridDim.x * blockDim.x;
    for (int k = 0; k < a.n; ++k) copy_bytes(a.peer_mb + slot + a.p[k].off, a.p[k].src, a.p[k].bytes, tid, nth);
    __threadfence_system();
    __syncthreads();
    if (threadIdx.x == 0 && atomicAdd((unsigned long long *)(a.my_flags + XF_CNT1), 1ull) == gridDim.x - 1) {
        a.my_flags[XF_CNT1] = 0;
        __threadfence_system();
        st_release_sys(a.peer_flags + XF_ARRIVED, s);
    }
    if (threadIdx.x == 0) {
        spin_until(a.my_flags + XF_ARRIVED, s);
        __threadfence();
    }
    __syncthreads();
    for (int k = 0; k < a.n; ++k) copy_bytes(a.p[k].dst, a.my_mb + slot + a.p[k].off, a.p[k].bytes, tid, nth);
    __threadfence_system();
    __syncthreads();
    if (threadIdx.x == 0 && atomicAdd((unsigned long long *)(a.my_flags + XF_CNT2), 1ull) == gridDim.x - 1) {
        a.my_flags[XF_CNT2] = 0;
        a.my_flags[XF_SEQ] = s;
        __threadfence_system();
        st_release_sys(a.peer_flags + XF_CONSUMED, s);
    }
}

static psml_status peer_exchange(psml_xport_s *x, int32_t n, const void *const *send, void *const *recv,
                                 const int64_t *bytes, cudaStream_t s) {
    if (!x->peer_mb) return fail(PSML_ERR_STATE, "peer transport not connected (psml_xport_peer_connect)");
    // pack the messages into mailbox windows of at most `cap` bytes; a larger exchange becomes
    // several rounds (both parties split identically: the message sizes are the same on both sides)
    XArgs a{};
    a.peer_mb = x->peer_mb; a.my_mb = x->my_mb; a.cap = x->cap; a.my_flags = x->my_flags; a.peer_flags = x->peer_flags;
    int64_t used = 0;
    auto flush = [&]() -> psml_status {
        if (a.n == 0) return PSML_OK;
        const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(64, (used + 65535) / 65536));
        xport_peer_kernel<<<grid, 512, 0, s>>>(a);
        PSML_LAUNCH_CHECK();
        a.n = 0;
        used = 0;
        return PSML_OK;
    };
    for (int k = 0; k < n; ++k) {
        int64_t done = 0;
        while (done < bytes[k]) {
            if (a.n == XMAX || used >= x->cap) PSML_TRY(flush());
            const int64_t len = std::min(bytes[k] - done, x->cap - used);
            XPiece &pc = a.p[a.n++];
            pc.src = (const uint8_t *)send[k] + done;
            pc.dst = (uint8_t *)recv[k] + done;
            pc.bytes = len;
            pc.off = used;
            used = (used + len + 255) & ~(int64_t)255;
            done += len;
        }
    }
    return flush();
}

}  // namespace psml

psml_status psml_xport_peer_create(int32_t party, int64_t capacity_bytes, psml_xport *out,
                                   uint8_t handle[PSML_PEER_HANDLE_BYTES]) {
    if (!out || !handle) return fail(PSML_ERR_INVALID, "null argument");
    if (party != 0 && party != 1) return fail(PSML_ERR_INVALID, "party must be 0 or 1");
    if (capacity_bytes < 4096) return fail(PSML_ERR_SHAPE, "capacity_bytes must be >= 4096");
    const int64_t cap = (capacity_bytes + 255) & ~(int64_t)255;
    int dev = 0;
    PSML_CUDA_TRY(cudaGetDevice(&dev));
    auto *x = new psml_xport_s;
    x->kind = 2;
    x->rank = party;
    x->device = dev;
    x->cap = cap;
    // two exchange slots + the fused kernels' window (PeerWindow), one allocation / one IPC handle
    if (cudaMalloc(&x->my_mb, 2 * cap + PW_BYTES) != cudaSuccess ||
        cudaMalloc(&x->my_flags, XF_WORDS * sizeof(uint64_t)) != cudaSuccess) {
        if (x->my_mb) cudaFree(x->my_mb);
        delete x;
        cudaGetLastError();
        return fail(PSML_ERR_NOMEM, "peer mailbox allocation failed");
    }
    if (cudaMemset(x->my_flags, 0, XF_WORDS * sizeof(uint64_t)) != cudaSuccess || cudaDeviceSynchronize() != cudaSuccess) {
        psml_xport_destroy(x);
        return fail(PSML_ERR_CUDA, "peer mailbox init failed");
    }
    PeerHandle h{};
    h.magic = PEER_MAGIC; h.version = 1; h.pid = (int64_t)getpid(); h.device = dev; h.party = party;
    h.raw_mb = (uint64_t)(uintptr_t)x->my_mb; h.raw_flags = (uint64_t)(uintptr_t)x->my_flags; h.cap = cap;
    if (cudaIpcGetMemHandle(&h.mb, x->my_mb) != cudaSuccess || cudaIpcGetMemHandle(&h.flags, x->my_flags) != cudaSuccess) {
        psml_xport_destroy(x);
        cudaGetLastError();
        return fail(PSML_ERR_CUDA, "cudaIpcGetMemHandle failed");
    }
    std::memset(handle, 0, PSML_PEER_HANDLE_BYTES);
    std::memcpy(handle, &h, sizeof(h));
    *out = x;
    return PSML_OK;
}

psml_status psml_xport_peer_connect(psml_xport x, const uint8_t peer_handle[PSML_PEER_HANDLE_BYTES]) {
    if (!x || !peer_handle) return fail(PSML_ERR_INVALID, "null argument");
    if (x->kind != 2) return fail(PSML_ERR_INVALID, "not a peer-memory transport");
    if (x->peer_mb) return fail(PSML_ERR_STATE, "already connected");
    PeerHandle h;
    std::memcpy(&h, peer_handle, sizeof(h));
    if (h.magic != PEER_MAGIC || h.version != 1) return fail(PSML_ERR_INVALID, "not a psml peer handle");
    if (h.party != 1 - x->rank) return fail(PSML_ERR_INVALID, "peer handle is not the other party's");
    if (h.cap != x->cap) return fail(PSML_ERR_SHAPE, "both parties must use the same mailbox capacity");
    if (h.pid == (int64_t)getpid()) {   // both parties in this process (one context): plain pointers
        x->peer_mb = (uint8_t *)(uintptr_t)h.raw_mb;
        x->peer_flags = (uint64_t *)(uintptr_t)h.raw_flags;
        return PSML_OK;
    }
    void *mb = nullptr, *fl = nullptr;
    cudaError_t e = cudaIpcOpenMemHandle(&mb, h.mb, cudaIpcMemLazyEnablePeerAccess);
    if (e == cudaSuccess) e = cudaIpcOpenMemHandle(&fl, h.flags, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) {
        if (mb) cudaIpcCloseMemHandle(mb);
        cudaGetLastError();
        return fail(PSML_ERR_CUDA, std::string("cudaIpcOpenMemHandle: ") + cudaGetErrorString(e));
    }
    x->peer_mb = (uint8_t *)mb;
    x->peer_flags = (uint64_t *)fl;
    x->peer_ipc = true;
    return PSML_OK;
}

psml_status psml_xport_destroy(psml_xport x) {
    if (!x) return PSML_OK;
    if (x->comm) ncclCommDestroy(x->comm);
    if (x->kind == 2) {
        cudaDeviceSynchronize();
        if (x->peer_ipc) {
            cudaIpcCloseMemHandle(x->peer_mb);
            cudaIpcCloseMemHandle(x->peer_flags);
        }
        if (x->my_mb) cudaFree(x->my_mb);
        if (x->my_flags) cudaFree(x->my_flags);
        cudaGetLastError();
    }
    delete x;
    return PSML_OK;
}

psml_status psml_xport_exchange(psml_xport x, int32_t n, const void *const *send, void *const *recv,
                                const int64_t *bytes, psml_stream stream) {
    if (!x) return fail(PSML_ERR_INVALID, "transport is null");
    if (n < 0 || (n > 0 && (!send || !recv || !bytes))) return fail(PSML_ERR_INVALID, "bad exchange list");
    int64_t tot = 0;
    for (int k = 0; k < n; ++k) {
        if (bytes[k] < 0) return fail(PSML_ERR_SHAPE, "negative message size");
        if (bytes[k] > 0 && (!send[k] || !recv[k])) return fail(PSML_ERR_INVALID, "null message buffer");
        tot += bytes[k];
    }
    if (tot == 0) return PSML_OK;
    cudaStream_t s = (cudaStream_t)stream;
    if (x->kind == 0) {
        const int peer = 1 - x->rank;
        ncclResult_t r = ncclGroupStart();
        if (r != ncclSuccess) return nccl_fail(r, "ncclGroupStart");
        for (int k = 0; k < n; ++k) {
            if (bytes[k] == 0) continue;
            r = ncclSend(send[k], (size_t)bytes[k], ncclUint8, peer, x->comm, s);
            if (r != ncclSuccess) { ncclGroupEnd(); return nccl_fail(r, "ncclSend"); }
            r = ncclRecv(recv[k], (size_t)bytes[k], ncclUint8, peer, x->comm, s);
            if (r != ncclSuccess) { ncclGroupEnd(); return nccl_fail(r, "ncclRecv"); }
        }
        r = ncclGroupEnd();
        if (r != ncclSuccess) return nccl_fail(r, "ncclGroupEnd");
    } else if (x->kind == 2) {
        PSML_TRY(peer_exchange(x, n, send, recv, bytes, s));
    } else {
        cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
        cudaStreamIsCapturing(s, &cs);
        if (cs != cudaStreamCaptureStatusNone)
            return fail(PSML_ERR_UNSUPPORTED, "a host-callback transport cannot be captured into a CUDA graph");
        const int32_t rc = x->fn(x->user, n, (void *const *)send, recv, bytes, stream);
        if (rc != 0) return fail(PSML_ERR_NCCL, "exchange callback returned " + std::to_string(rc));
    }
    x->bytes_sent += tot;
    x->exchanges += 1;
    return PSML_OK;
}

// ------------------------------------------------------------------------------------------------
// data-parallel communicator of one party (per-party uint64 all-reduce of the
// untruncated gradient shares over the party's GPUs)
// ------------------------------------------------------------------------------------------------
struct psml_dp_s {
    ncclComm_t comm = nullptr;
    int rank = 0, size = 1;
};

psml_status psml_dp_create(const uint8_t uid[128], int32_t rank, int32_t size, psml_dp *out) {
    if (!out) return fail(PSML_ERR_INVALID, "null argument");
    if (size < 1 || rank < 0 || rank >= size) return fail(PSML_ERR_INVALID, "need 0 <= rank < size");
    auto *d = new psml_dp_s;
    d->rank = rank;
    d->size = size;
    if (size > 1) {
        if (!uid) { delete d; return fail(PSML_ERR_INVALID, "uid is null"); }
        ncclUniqueId id;
        std::memcpy(&id, uid, sizeof(id));
        ncclResult_t r = ncclCommInitRank(&d->comm, size, id, rank);
        if (r != ncclSuccess) { delete d; return nccl_fail(r, "ncclCommInitRank (dp)"); }
    }
    *out = d;
    return PSML_OK;
}

psml_status psml_dp_destroy(psml_dp d) {
    if (!d) return PSML_OK;
    if (d->comm) ncclCommDestroy(d->comm);
    delete d;
    return PSML_OK;
}

psml_status psml_dp_size(psml_dp d, int32_t *size) {
    if (!d || !size) return fail(PSML_ERR_INVALID, "null argument");
    *size = d->size;
    return PSML_OK;
}

psml_status psml_dp_allreduce(psml_dp d, void *buf, int64_t n, int32_t l, psml_stream stream) {
    if (!d) return fail(PSML_ERR_INVALID, "dp is null");
    if (l != 32 && l != 64) return fail(PSML_ERR_INVALID, "l must be 32 or 64");
    if (n < 0) return fail(PSML_ERR_SHAPE, "n < 0");
    if (d->size == 1 || n == 0) return PSML_OK;
    if (!buf) return fail(PSML_ERR_INVALID, "buf is null");
    // Z_{2^l} addition is unsigned wraparound addition: exactly ncclSum on ncclUint64 / ncclUint32
    ncclResult_t r = ncclAllReduce(buf, buf, (size_t)n, l == 64 ? ncclUint64 : ncclUint32, ncclSum, d->comm,
                                   (cudaStream_t)stream);
    if (r != ncclSuccess) return nccl_fail(r, "ncclAllReduce");
    return PSML_OK;
}

namespace psml {
void xport_account(psml_xport x, int64_t exchanges, int64_t bytes) {
    if (!x) return;
    x->exchanges += exchanges;
    x->bytes_sent += bytes;
}

bool xport_peer_window(psml_xport x, PeerWindow *w) {
    if (!x || x->kind != 2 || !x->peer_mb || !w) return false;
    w->my_win = x->my_mb + 2 * x->cap;
    w->peer_win = x->peer_mb + 2 * x->cap;
    w->bytes = PW_BYTES;
    w->my_flags = x->my_flags;
    w->peer_flags = x->peer_flags;
    return true;
}
}  // namespace psml

psml_status psml_xport_stats(psml_xport x, int64_t *bytes_sent, int64_t *exchanges) {
    if (!x) return fail(PSML_ERR_INVALID, "transport is null");
    if (bytes_sent) *bytes_sent = x->bytes_sent;
    if (exchanges) *exchanges = x->exchanges;
    return PSML_OK;
}
