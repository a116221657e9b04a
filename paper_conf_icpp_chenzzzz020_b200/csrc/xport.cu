// xport.cu -- transports of the split deployment (include/psml.h "Split deployment").
//
// PAPER.md Fig. 1b (L55-L61) puts the two servers on different machines and L65 has them
// "compute E and F via communication": every opening is one symmetric exchange of the parties'
// masked messages (R5).  Two transports implement that exchange:
//   NCCL      a library-owned 2-rank communicator per party pair; one exchange = one grouped
//             ncclSend/ncclRecv per buffer on the step's stream (stream-ordered, NVLink P2P
//             between GPUs, no host synchronisation);
//   callback  a host function supplied by the caller (host-staged gloo in the tests, where both
//             parties' processes share one GPU and NCCL refuses duplicate devices).
#include <nccl.h>

#include <cstring>
#include <string>

#include "common.cuh"

struct psml_xport_s {
    int kind = 0;                 // 0 NCCL, 1 callback
    ncclComm_t comm = nullptr;
    int rank = 0;
    psml_exchange_fn fn = nullptr;
    void *user = nullptr;
    int64_t bytes_sent = 0, exchanges = 0;
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

psml_status psml_xport_destroy(psml_xport x) {
    if (!x) return PSML_OK;
    if (x->comm) ncclCommDestroy(x->comm);
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
    } else {
        const int32_t rc = x->fn(x->user, n, (void *const *)send, recv, bytes, stream);
        if (rc != 0) return fail(PSML_ERR_NCCL, "exchange callback returned " + std::to_string(rc));
    }
    x->bytes_sent += tot;
    x->exchanges += 1;
    return PSML_OK;
}

psml_status psml_xport_stats(psml_xport x, int64_t *bytes_sent, int64_t *exchanges) {
    if (!x) return fail(PSML_ERR_INVALID, "transport is null");
    if (bytes_sent) *bytes_sent = x->bytes_sent;
    if (exchanges) *exchanges = x->exchanges;
    return PSML_OK;
}
