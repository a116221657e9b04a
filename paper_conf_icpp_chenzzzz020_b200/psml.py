"""Thin ctypes binding of libpsml.so (include/psml.h).  Argument marshalling only: every step of
the hot path runs in the library's CUDA kernels.  PyTorch supplies device memory and streams.

There is no CPU fallback: importing works anywhere (so the CPU test suite can check the
exported symbols), but every compute call raises if the library or a CUDA device is missing.
Function names follow the C ABI without the ``psml_`` prefix.
"""
import ctypes
import os

import torch

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "libpsml.so")
HEADER = os.path.join(os.path.dirname(HERE), "include", "psml.h")

STATUS = {0: "PSML_OK", 1: "PSML_ERR_INVALID", 2: "PSML_ERR_SHAPE", 3: "PSML_ERR_ALIGN",
          4: "PSML_ERR_UNSUPPORTED", 5: "PSML_ERR_CUDA", 6: "PSML_ERR_NOMEM", 7: "PSML_ERR_STATE",
          8: "PSML_ERR_NCCL"}
TRANS_A, TRANS_B, PAPER_FORM = 1, 2, 4
LINREG, LOGREG, MLP, CNN, SVM, RNN = 0, 1, 2, 3, 4, 5

vp, i32, i64, u32, u64 = (ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_uint32,
                          ctypes.c_uint64)
P2 = vp * 2


class PsmlError(RuntimeError):
    def __init__(self, fn, status, msg):
        super().__init__(f"{fn}: {STATUS.get(status, status)}: {msg}")
        self.status = status


class Ring(ctypes.Structure):
    _fields_ = [("l", i32), ("frac_bits", i32)]


class Options(ctypes.Structure):
    """psml_options (include/psml.h): explicit per-context execution options."""
    _fields_ = [(n, i32) for n in ("seg_backend", "pdl", "fused_open", "fused_step", "fused_dealer",
                                    "deal_split", "deal_after", "gradw_branch", "simt_cluster",
                                    "rows_kernel", "msb_chain", "conv_gw", "split_fused", "deal_on_launch",
                                    "tc_small")]


# Test-harness convenience of the BINDING (the library reads no environment): PSML_* variables
# override the defaults of every context this process creates, so a subprocess test can select an
# alternative implementation; the values map to explicit psml_options fields.
_ENV_OPTIONS = {
    "PSML_SEG": ("seg_backend", {"simt": 1, "tc": 2}),
    "PSML_PDL": ("pdl", {"0": 0, "1": 1}),
    "PSML_OPEN": ("fused_open", {"fused": 1, "mask": 0}),
    "PSML_FUSE": ("fused_step", {"0": 0, "1": 1}),
    "PSML_DEAL": ("fused_dealer", {"items": 0, "fused": 1}),
    "PSML_DEAL_SPLIT": ("deal_split", {"0": 0, "1": 1}),
    "PSML_DEAL_AFTER": ("deal_after", None),
    "PSML_GRADW_BRANCH": ("gradw_branch", {"0": 0, "1": 1}),
    "PSML_SIMT": ("simt_cluster", {"small": 0, "cluster": 1}),
    "PSML_ROWS": ("rows_kernel", {"0": 0, "1": 1}),
    "PSML_MSB_CHAIN": ("msb_chain", {"rounds": 1, "pair": 0}),
    "PSML_CONV_GW": ("conv_gw", {"generic": 0, "image": 1}),
    "PSML_SPLIT_FUSED": ("split_fused", {"0": 0, "1": 1}),
    "PSML_DEAL_ON_LAUNCH": ("deal_on_launch", {"0": 0, "1": 1}),
    "PSML_TC_SMALL": ("tc_small", {"0": 0, "1": 1, "2": 2}),
}


def default_options(**overrides):
    o = Options()
    _call("psml_options_default", ctypes.byref(o))
    for var, (field, table) in _ENV_OPTIONS.items():
        v = os.environ.get(var)
        if v is not None:
            setattr(o, field, int(v) if table is None else table.get(v, getattr(o, field)))
    for k, v in overrides.items():
        setattr(o, k, v)
    return o


class Trace(ctypes.Structure):
    _fields_ = [("E", vp * 2), ("E_open", vp), ("F", vp * 2), ("F_open", vp)]


class ModelDesc(ctypes.Structure):
    _fields_ = [("kind", i32), ("n_layers", i32), ("dims", i64 * 8), ("batch", i32),
                ("lr_shift", i32), ("master_frac_bits", i32), ("dealer_seed", u64),
                ("pair_id", u32), ("cnn_c", i32), ("cnn_h", i32), ("cnn_w", i32), ("cnn_k", i32),
                ("cnn_cout", i32), ("cnn_hidden", i32), ("cnn_classes", i32),
                ("fwd_frac_bits", i32 * 8), ("compare", i32), ("weight_decay_shift", i32),
                ("rnn_steps", i32), ("mask_reuse", i32), ("deal_role", i32),
                ("strong_pairs", i32)]


# psml_exchange_fn (include/psml.h): (user, n, send[], recv[], bytes[], stream) -> 0 on success
EXCHANGE_FN = ctypes.CFUNCTYPE(i32, vp, i32, ctypes.POINTER(vp), ctypes.POINTER(vp),
                               ctypes.POINTER(i64), vp)

# name -> (restype, argtypes); mirrors include/psml.h
_SIGS = {
    "psml_abi_version": (i32, []),
    "psml_last_error": (ctypes.c_char_p, []),
    "psml_device_info": (i32, [vp, vp, vp]),
    "psml_kernel_launch_count": (u64, []),
    "psml_prof_enable": (i32, [i32]),
    "psml_prof_read": (i32, [vp, vp, vp]),
    "psml_bench_mac_peak": (i32, [i32, vp]),
    "psml_ctx_create": (i32, [Ring, i32, vp]),
    "psml_ctx_destroy": (i32, [vp]),
    "psml_options_default": (i32, [vp]),
    "psml_ctx_set_options": (i32, [vp, vp]),
    "psml_prg_fill": (i32, [Ring, u64, u32, u64, u64, i64, vp, vp]),
    "psml_encode": (i32, [Ring, vp, i64, vp, vp]),
    "psml_decode": (i32, [Ring, vp, i64, vp, vp]),
    "psml_share": (i32, [Ring, u64, u64, vp, i64, vp, vp, vp]),
    "psml_reconstruct": (i32, [Ring, vp, vp, i64, vp, vp]),
    "psml_encode_share": (i32, [Ring, u64, u64, vp, i64, vp, vp, vp]),
    "psml_encode_share_u8": (i32, [Ring, u64, u64, vp, i64, ctypes.c_double, vp, vp, vp]),
    "psml_encode_share_onehot": (i32, [Ring, u64, u64, vp, i64, i64, vp, vp, vp]),
    "psml_triplet_gen": (i32, [vp, u64, u64, i64, i64, i64, P2, P2, P2, vp]),
    "psml_triplet_gen_rows": (i32, [vp, u64, u64, i64, i64, i64, i64, i64, P2, P2, P2, vp]),
    "psml_hadamard_triplet_gen": (i32, [Ring, u64, u64, i64, P2, P2, P2, vp]),
    "psml_msb_material_words": (i64, [Ring, i64]),
    "psml_msb_dealer": (i32, [Ring, u64, u64, i64, P2, vp]),
    "psml_secure_matmul": (i32, [vp, P2, P2, P2, P2, P2, i64, i64, i64, i32, i32, P2, vp, vp]),
    "psml_secure_hadamard": (i32, [vp, P2, P2, P2, P2, P2, i64, i32, P2, vp]),
    "psml_beaver_mask": (i32, [vp, i32, vp, vp, vp, vp, i64, i64, i64, i32, vp, vp, vp]),
    "psml_beaver_open_matmul": (i32, [vp, i32, vp, vp, vp, vp, vp, vp, vp, i64, i64, i64, i32, vp, vp]),
    "psml_truncate": (i32, [Ring, i32, vp, i64, i32, vp]),
    "psml_secure_msb": (i32, [vp, P2, i64, P2, P2, vp, vp]),
    "psml_secure_relu": (i32, [vp, P2, i64, P2, P2, P2, P2, P2, vp, vp]),
    "psml_secure_eq9": (i32, [vp, P2, i64, P2, P2, P2, P2, P2, vp]),
    "psml_ring_gemm": (i32, [vp, vp, vp, i64, i64, i64, vp, vp]),
    "psml_delta_encode": (i32, [vp, vp, vp, i64, i64, vp, vp, vp, vp, vp, vp, vp]),
    "psml_delta_apply": (i32, [vp, i64, i64, i32, vp, vp, vp, vp, vp, vp]),
    "psml_model_create": (i32, [vp, ctypes.POINTER(ModelDesc), vp]),
    "psml_model_destroy": (i32, [vp]),
    "psml_model_layer_shape": (i32, [vp, i32, vp, vp]),
    "psml_model_set_master": (i32, [vp, i32, P2, vp]),
    "psml_model_get_master": (i32, [vp, i32, P2, vp]),
    "psml_model_deal": (i32, [vp, u32, i32, vp]),
    "psml_secure_train_step": (i32, [vp, P2, P2, u32, vp]),
    "psml_train_forward_backward": (i32, [vp, P2, P2, u32, vp]),
    "psml_model_output": (i32, [vp, vp, vp, vp]),
    "psml_model_grads": (i32, [vp, vp, vp]),
    "psml_train_apply_update": (i32, [vp, i32, vp]),
    "psml_secure_infer": (i32, [vp, P2, u32, P2, vp]),
    "psml_model_capture_step": (i32, [vp, P2, P2, i32, vp]),
    "psml_model_step_graph": (i32, [vp, u32, vp]),
    "psml_model_step_host": (i32, [vp, vp, vp, i32, u64, u32, vp, vp]),
    "psml_model_step_device": (i32, [vp, vp, vp, u64, u32, vp]),
    "psml_model_graph_nodes": (i32, [vp, vp]),
    "psml_nccl_unique_id": (i32, [vp]),
    "psml_xport_nccl_create": (i32, [vp, i32, vp]),
    "psml_xport_callback_create": (i32, [EXCHANGE_FN, vp, vp]),
    "psml_xport_destroy": (i32, [vp]),
    "psml_xport_exchange": (i32, [vp, i32, vp, vp, vp, vp]),
    "psml_xport_stats": (i32, [vp, vp, vp]),
    "psml_party_forward_backward": (i32, [vp, i32, vp, vp, vp, u32, vp]),
    "psml_party_apply_update": (i32, [vp, i32, i32, vp]),
    "psml_xport_peer_create": (i32, [i32, i64, vp, vp]),
    "psml_xport_peer_connect": (i32, [vp, vp]),
    "psml_dp_create": (i32, [vp, i32, i32, vp]),
    "psml_dp_destroy": (i32, [vp]),
    "psml_dp_size": (i32, [vp, vp]),
    "psml_dp_allreduce": (i32, [vp, vp, i64, i32, vp]),
    "psml_party_train_step": (i32, [vp, i32, vp, vp, vp, vp, u32, vp]),
    "psml_ctx_create_party": (i32, [Ring, i32, i32, vp, vp, vp]),
    "psml_secure_matmul_party": (i32, [vp, vp, vp, vp, vp, vp, i64, i64, i64, i32, i32, vp, vp]),
    "psml_dealer_party_seed": (u64, [u64, i32]),
    "psml_model_deal_bundle": (i32, [vp, u32, i32, vp, vp, vp]),
    "psml_model_deal_party": (i32, [vp, u32, i32, vp, i64, vp]),
    "psml_fss_material_words": (i64, [Ring, i64]),
    "psml_fss_dealer": (i32, [Ring, u64, u64, i64, P2, vp]),
    "psml_secure_drelu_fss": (i32, [vp, P2, i64, P2, P2, vp, vp]),
    "psml_secure_relu_fss": (i32, [vp, P2, i64, P2, P2, P2, P2, P2, P2, vp]),
    "psml_fss_mask": (i32, [vp, i32, vp, i64, vp, vp, vp]),
    "psml_fss_open_drelu": (i32, [vp, i32, vp, vp, i64, vp, vp, vp]),
    "psml_party_capture_step": (i32, [vp, i32, vp, vp, vp, vp, i32, vp]),
}
PEER_HANDLE_BYTES = 256
EXPORTS = tuple(_SIGS)

_lib = None


def lib():
    """Load libpsml.so (build it first with paper_conf_icpp_chenzzzz020_b200.build)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise PsmlError("load", 4, f"{LIB_PATH} missing: run `python -m "
                            "paper_conf_icpp_chenzzzz020_b200.build` (no CPU fallback exists)")
        L = ctypes.CDLL(LIB_PATH)
        for name, (res, args) in _SIGS.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def _call(name, *args):
    st = getattr(lib(), name)(*args)
    if st != 0:
        raise PsmlError(name, st, lib().psml_last_error().decode(errors="replace"))


# ---------------------------------------------------------------------------------------------
# marshalling helpers
# ---------------------------------------------------------------------------------------------
def dtype_of(l):
    return torch.uint64 if l == 64 else torch.uint32


def _host_ptr(t):
    """Address of a contiguous CPU tensor (pinned for asynchronous copies)."""
    if t.is_cuda or not t.is_contiguous():
        raise PsmlError("marshal", 1, "host tensor must be a contiguous CPU tensor")
    return ctypes.c_void_p(t.data_ptr())


def _ptr(t):
    if t is None:
        return None
    if not t.is_cuda:
        raise PsmlError("marshal", 1, "tensor must be on a CUDA device")
    if not t.is_contiguous():
        raise PsmlError("marshal", 1, "tensor must be contiguous")
    return ctypes.c_void_p(t.data_ptr())


def _pair(ts):
    """A pair of device pointers; every tensor must be a contiguous CUDA tensor (no CPU fallback,
    and the C ABI takes sizes from its own arguments, so a wrong tensor must not reach it)."""
    if ts is None:
        return None
    return P2(*(None if t is None else _ptr(t).value for t in ts))


def _check(ts, words, dtypes, what):
    """Shape / dtype guard for model-sized buffers (the ABI reads `words` elements from each)."""
    for t in ([ts] if torch.is_tensor(ts) else list(ts)):
        if t is None:
            continue
        if t.dtype not in dtypes:
            raise PsmlError("marshal", 1, f"{what}: dtype {t.dtype}, expected one of {dtypes}")
        if t.numel() != words:
            raise PsmlError("marshal", 2, f"{what}: {t.numel()} elements, expected {words}")


def _stream(stream=None):
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def empty(n, l, like_shape=None):
    shape = like_shape if like_shape is not None else (n,)
    return torch.empty(shape, dtype=dtype_of(l), device="cuda")


def empty_pair(shape, l):
    return (torch.empty(shape, dtype=dtype_of(l), device="cuda"),
            torch.empty(shape, dtype=dtype_of(l), device="cuda"))


def tag(s):
    b = (s.encode() if isinstance(s, str) else bytes(s)) + b"\0\0\0\0"
    return int.from_bytes(b[:4], "little")


# ---------------------------------------------------------------------------------------------
# library / device
# ---------------------------------------------------------------------------------------------
def abi_version():
    return lib().psml_abi_version()


def kernel_launch_count():
    return lib().psml_kernel_launch_count()


PROF_GEMM, PROF_TC, PROF_MSB, PROF_HAD, PROF_DEALER, PROF_MASK = range(6)


def bench_mac_peak(l=64):
    """Measured ring multiply-add throughput on CUDA cores (psml_bench_mac_peak), ring MACs/s."""
    v = ctypes.c_double()
    _call("psml_bench_mac_peak", l, ctypes.byref(v))
    return v.value


def dealer_party_seed(dealer_seed, party):
    """s_i = PRG(dealer seed, "KD", i)[0]: the only dealer secret party i holds (R23)."""
    return lib().psml_dealer_party_seed(dealer_seed, party)


def prof_enable(cls):
    """Time every library launch of kernel class `cls` with CUDA events (-1 disables)."""
    _call("psml_prof_enable", cls)


def prof_read():
    """(total ms, launches, algorithmic work) of the profiled class since the last read."""
    ms, n, w = ctypes.c_double(), i64(), ctypes.c_double()
    _call("psml_prof_read", ctypes.byref(ms), ctypes.byref(n), ctypes.byref(w))
    return ms.value, n.value, w.value


def device_info():
    a, b, c = i32(), i32(), i32()
    _call("psml_device_info", ctypes.byref(a), ctypes.byref(b), ctypes.byref(c))
    return a.value, b.value, c.value


class Ctx:
    """psml_ctx: one per GPU and host thread.  backend: 0 auto, 1 CUDA-core, 2 tcgen05."""

    def __init__(self, l=64, frac_bits=13, backend=0, party=None, xport=None, dp=None, options=None):
        """party/xport/dp: a per-party context (psml_ctx_create_party) for psml_secure_matmul_party;
        options: psml_options overrides (dict), on top of the defaults (default_options)."""
        self.ring = Ring(l, frac_bits)
        self.l = l
        self.party = party
        self._keep = (xport, dp)   # the transport / communicator must outlive the context
        h = vp()
        if party is None:
            _call("psml_ctx_create", self.ring, backend, ctypes.byref(h))
        else:
            _call("psml_ctx_create_party", self.ring, backend, party, xport.handle, dp.handle if dp else None,
                  ctypes.byref(h))
        self.handle = h
        self.options = default_options(**(options or {}))
        _call("psml_ctx_set_options", self.handle, ctypes.byref(self.options))

    def close(self):
        if self.handle:
            lib().psml_ctx_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


# ---------------------------------------------------------------------------------------------
# client / dealer
# ---------------------------------------------------------------------------------------------
def prg_fill(ring, seed, tag_value, call_id, n, offset=0, out=None, stream=None):
    out = out if out is not None else empty(n, ring.l)
    _call("psml_prg_fill", ring, seed, tag_value, call_id, offset, n, _ptr(out), _stream(stream))
    return out


def encode(ring, x, stream=None):
    x = x.to(dtype=torch.float64, device="cuda").contiguous()
    v = torch.empty(x.shape, dtype=dtype_of(ring.l), device="cuda")
    _call("psml_encode", ring, _ptr(x), x.numel(), _ptr(v), _stream(stream))
    return v


def decode(ring, v, stream=None):
    x = torch.empty(v.shape, dtype=torch.float64, device="cuda")
    _call("psml_decode", ring, _ptr(v), v.numel(), _ptr(x), _stream(stream))
    return x


def share(ring, seed, stream_id, x, out=None, stream=None):
    x0, x1 = out if out is not None else empty_pair(x.shape, ring.l)
    _call("psml_share", ring, seed, stream_id, _ptr(x), x.numel(), _ptr(x0), _ptr(x1),
          _stream(stream))
    return x0, x1


def encode_share(ring, seed, stream_id, x, out=None, stream=None):
    """psml_encode + psml_share in one kernel (x: float64 device tensor)."""
    if x.dtype != torch.float64:
        raise PsmlError("marshal", 1, "encode_share takes float64")
    x0, x1 = out if out is not None else empty_pair(x.shape, ring.l)
    _call("psml_encode_share", ring, seed, stream_id, _ptr(x), x.numel(), _ptr(x0), _ptr(x1),
          _stream(stream))
    return x0, x1


def encode_share_u8(ring, seed, stream_id, q, den=255.0, out=None, stream=None):
    """encode_share of q / den from bytes (q: uint8 device tensor, e.g. 8-bit pixels)."""
    if q.dtype != torch.uint8:
        raise PsmlError("marshal", 1, "encode_share_u8 takes uint8")
    q = q.contiguous()
    x0, x1 = out if out is not None else empty_pair(q.shape, ring.l)
    _call("psml_encode_share_u8", ring, seed, stream_id, _ptr(q), q.numel(), float(den), _ptr(x0), _ptr(x1),
          _stream(stream))
    return x0, x1


def encode_share_onehot(ring, seed, stream_id, cls, classes, out=None, stream=None):
    """encode_share of the one-hot (rows x classes) matrix of class indices cls (uint8 device)."""
    if cls.dtype != torch.uint8:
        raise PsmlError("marshal", 1, "encode_share_onehot takes uint8 class indices")
    cls = cls.contiguous()
    x0, x1 = out if out is not None else empty_pair((cls.numel(), classes), ring.l)
    _call("psml_encode_share_onehot", ring, seed, stream_id, _ptr(cls), cls.numel(), classes, _ptr(x0),
          _ptr(x1), _stream(stream))
    return x0, x1


def reconstruct(ring, x0, x1, stream=None):
    x = torch.empty_like(x0)
    _call("psml_reconstruct", ring, _ptr(x0), _ptr(x1), x0.numel(), _ptr(x), _stream(stream))
    return x


def triplet_gen(ctx, seed, call_id, M, K, N, stream=None):
    U, V, Z = empty_pair((M, K), ctx.l), empty_pair((K, N), ctx.l), empty_pair((M, N), ctx.l)
    _call("psml_triplet_gen", ctx.handle, seed, call_id, M, K, N, _pair(U), _pair(V), _pair(Z),
          _stream(stream))
    return U, V, Z


def triplet_gen_rows(ctx, seed, call_id, M_total, row0, M, K, N, stream=None):
    """Rows [row0, row0 + M) of triplet_gen(seed, call_id, M_total, K, N): U / Z row blocks and the
    whole V (the M-row sharding of a secure product over pairs, R28)."""
    U, V, Z = empty_pair((M, K), ctx.l), empty_pair((K, N), ctx.l), empty_pair((M, N), ctx.l)
    _call("psml_triplet_gen_rows", ctx.handle, seed, call_id, M_total, row0, M, K, N, _pair(U), _pair(V), _pair(Z),
          _stream(stream))
    return U, V, Z


def hadamard_triplet_gen(ring, seed, call_id, n, stream=None):
    U, V, Z = empty_pair(n, ring.l), empty_pair(n, ring.l), empty_pair(n, ring.l)
    _call("psml_hadamard_triplet_gen", ring, seed, call_id, n, _pair(U), _pair(V), _pair(Z),
          _stream(stream))
    return U, V, Z


def msb_material_words(ring, n):
    return lib().psml_msb_material_words(ring, n)


def msb_dealer(ring, seed, call_id, n, stream=None):
    mat = empty_pair(msb_material_words(ring, n), ring.l)
    _call("psml_msb_dealer", ring, seed, call_id, n, _pair(mat), _stream(stream))
    return mat


# ---------------------------------------------------------------------------------------------
# server side
# ---------------------------------------------------------------------------------------------
def secure_matmul(ctx, A, B, U, V, Z, M, K, N, flags=0, trunc=0, out=None, trace=False,
                  stream=None):
    C = out if out is not None else empty_pair((M, N), ctx.l)
    tr = None
    tr_t = None
    if trace:
        tr_t = dict(E0=empty(0, ctx.l, (M, K)), E1=empty(0, ctx.l, (M, K)), E=empty(0, ctx.l, (M, K)),
                    F0=empty(0, ctx.l, (K, N)), F1=empty(0, ctx.l, (K, N)), F=empty(0, ctx.l, (K, N)))
        tr = Trace(P2(tr_t["E0"].data_ptr(), tr_t["E1"].data_ptr()), tr_t["E"].data_ptr(),
                   P2(tr_t["F0"].data_ptr(), tr_t["F1"].data_ptr()), tr_t["F"].data_ptr())
    _call("psml_secure_matmul", ctx.handle, _pair(A), _pair(B), _pair(U), _pair(V), _pair(Z),
          M, K, N, flags, trunc, _pair(C), ctypes.byref(tr) if tr is not None else None,
          _stream(stream))
    return (C, tr_t) if trace else C


def secure_matmul_party(ctx, A_i, B_i, U_i, V_i, Z_i, M, K, N, flags=0, trunc=0, out=None, stream=None):
    """Collective one-party Beaver product through the ctx's pair transport (per-party ctx)."""
    C = out if out is not None else torch.empty((M, N), dtype=dtype_of(ctx.l), device="cuda")
    _call("psml_secure_matmul_party", ctx.handle, _ptr(A_i), _ptr(B_i), _ptr(U_i), _ptr(V_i), _ptr(Z_i), M, K, N,
          flags, trunc, _ptr(C), _stream(stream))
    return C


def beaver_mask(ctx, party, A_i, B_i, U_i, V_i, M, K, N, flags=0, stream=None):
    """Split deployment, round 1 of party `party`: returns its send buffers (E_i, F_i)."""
    E = empty(0, ctx.l, (M, K))
    F = empty(0, ctx.l, (K, N))
    _call("psml_beaver_mask", ctx.handle, party, _ptr(A_i), _ptr(B_i), _ptr(U_i), _ptr(V_i), M, K, N,
          flags, _ptr(E), _ptr(F), _stream(stream))
    return E, F


def beaver_open_matmul(ctx, party, E_send, E_recv, F_send, F_recv, U_i, V_i, Z_i, M, K, N, trunc=0,
                       out=None, stream=None):
    """Split deployment, round 2 of party `party`: its share C_i of A.B (Eq. 8 shape)."""
    C = out if out is not None else empty(0, ctx.l, (M, N))
    _call("psml_beaver_open_matmul", ctx.handle, party, _ptr(E_send), _ptr(E_recv), _ptr(F_send),
          _ptr(F_recv), _ptr(U_i), _ptr(V_i), _ptr(Z_i), M, K, N, trunc, _ptr(C), _stream(stream))
    return C


def secure_hadamard(ctx, A, B, U, V, Z, trunc=0, out=None, stream=None):
    n = A[0].numel()
    C = out if out is not None else empty_pair(A[0].shape, ctx.l)
    _call("psml_secure_hadamard", ctx.handle, _pair(A), _pair(B), _pair(U), _pair(V), _pair(Z), n,
          trunc, _pair(C), _stream(stream))
    return C


def truncate(ring, party, x, bits, stream=None):
    _call("psml_truncate", ring, party, _ptr(x), x.numel(), bits, _stream(stream))
    return x


def secure_msb(ctx, x, mat, want_bool=False, stream=None):
    n = x[0].numel()
    a = empty_pair(x[0].shape, ctx.l)
    b = empty_pair(x[0].shape, ctx.l) if want_bool else None
    _call("psml_secure_msb", ctx.handle, _pair(x), n, _pair(mat), _pair(a), _pair(b),
          _stream(stream))
    return (a, b) if want_bool else a


def secure_relu(ctx, x, mat, U, V, Z, stream=None):
    n = x[0].numel()
    y, d = empty_pair(x[0].shape, ctx.l), empty_pair(x[0].shape, ctx.l)
    _call("psml_secure_relu", ctx.handle, _pair(x), n, _pair(mat), _pair(U), _pair(V), _pair(Z),
          _pair(y), _pair(d), _stream(stream))
    return y, d


def fss_dealer(ring, seed, call_id, n, stream=None):
    """One-round FSS comparison material (psml_fss_dealer, R22): 257 n words per party."""
    w = lib().psml_fss_material_words(ring, n)
    if w < 0:
        raise PsmlError("psml_fss_material_words", 4, "the FSS comparison is built for Z_2^64")
    mat = empty_pair(w, ring.l)
    _call("psml_fss_dealer", ring, seed, call_id, n, _pair(mat), _stream(stream))
    return mat


def secure_drelu_fss(ctx, x, mat, trace=False, stream=None):
    n = x[0].numel()
    d = empty_pair(x[0].shape, ctx.l)
    xh = empty(n, ctx.l) if trace else None
    _call("psml_secure_drelu_fss", ctx.handle, _pair(x), n, _pair(mat), _pair(d), _ptr(xh), _stream(stream))
    return (d, xh) if trace else d


def secure_relu_fss(ctx, x, mat, U, V, Z, stream=None):
    n = x[0].numel()
    y, d = empty_pair(x[0].shape, ctx.l), empty_pair(x[0].shape, ctx.l)
    _call("psml_secure_relu_fss", ctx.handle, _pair(x), n, _pair(mat), _pair(U), _pair(V), _pair(Z),
          _pair(y), _pair(d), _stream(stream))
    return y, d


def fss_mask(ctx, party, x_i, mat_i, stream=None):
    n = x_i.numel()
    msg = empty(n, ctx.l)
    _call("psml_fss_mask", ctx.handle, party, _ptr(x_i), n, _ptr(mat_i), _ptr(msg), _stream(stream))
    return msg


def fss_open_drelu(ctx, party, msg_send, msg_recv, mat_i, stream=None):
    n = msg_send.numel()
    d = empty(n, ctx.l)
    _call("psml_fss_open_drelu", ctx.handle, party, _ptr(msg_send), _ptr(msg_recv), n, _ptr(mat_i), _ptr(d),
          _stream(stream))
    return d


def secure_eq9(ctx, x, mat, U, V, Z, stream=None):
    n = x[0].numel()
    y = empty_pair(x[0].shape, ctx.l)
    _call("psml_secure_eq9", ctx.handle, _pair(x), n, _pair(mat), _pair(U), _pair(V), _pair(Z),
          _pair(y), _stream(stream))
    return y


def ring_gemm(ctx, A, B, out=None, stream=None):
    M, K = A.shape
    N = B.shape[1]
    C = out if out is not None else empty(0, ctx.l, (M, N))
    _call("psml_ring_gemm", ctx.handle, _ptr(A), _ptr(B), M, K, N, _ptr(C), _stream(stream))
    return C


def delta_encode(ctx, cur, prev, stream=None):
    rows, cols = cur.shape
    row_ptr = torch.empty(rows + 1, dtype=torch.int32, device="cuda")
    col_idx = torch.empty(rows * cols, dtype=torch.int32, device="cuda")
    vals = empty(rows * cols, ctx.l)
    dense = empty(0, ctx.l, (rows, cols))
    nnz, is_csr = i64(), i32()
    _call("psml_delta_encode", ctx.handle, _ptr(cur), _ptr(prev), rows, cols, _ptr(row_ptr),
          _ptr(col_idx), _ptr(vals), _ptr(dense), ctypes.byref(nnz), ctypes.byref(is_csr),
          _stream(stream))
    if is_csr.value:
        return dict(is_csr=True, nnz=nnz.value, row_ptr=row_ptr, col_idx=col_idx[:nnz.value],
                    vals=vals[:nnz.value])
    return dict(is_csr=False, nnz=nnz.value, dense=dense)


def delta_apply(ctx, target, enc, stream=None):
    rows, cols = target.shape
    if enc["is_csr"]:
        _call("psml_delta_apply", ctx.handle, rows, cols, 1, _ptr(enc["row_ptr"]),
              _ptr(enc["col_idx"]), _ptr(enc["vals"]) if enc["nnz"] else None, None, _ptr(target),
              _stream(stream))
    else:
        _call("psml_delta_apply", ctx.handle, rows, cols, 0, None, None, None, _ptr(enc["dense"]),
              _ptr(target), _stream(stream))
    return target


# ---------------------------------------------------------------------------------------------
# models
# ---------------------------------------------------------------------------------------------
class Model:
    """psml_model: weight shares, dealer pool and workspaces of one secure model."""

    def __init__(self, ctx, kind, dims=None, batch=128, lr_shift=14, master_frac_bits=27,
                 dealer_seed=0x50534D4C + 2, pair_id=0, cnn=(3, 32, 32, 5, 16, 64, 10),
                 fwd_frac_bits=None, compare=0, weight_decay_shift=0, rnn_steps=0, deal_role=0,
                 mask_reuse=False, strong_pairs=0):
        d = ModelDesc()
        d.kind = kind
        dims = list(dims or ([784, 1] if kind in (LINREG, LOGREG, SVM) else [784, 128, 128, 10]))
        d.n_layers = 3 if kind == CNN else (2 if kind == RNN else len(dims) - 1)
        for i, v in enumerate(dims[:8]):
            d.dims[i] = v
        d.batch, d.lr_shift, d.master_frac_bits = batch, lr_shift, master_frac_bits
        d.dealer_seed, d.pair_id = dealer_seed, pair_id
        (d.cnn_c, d.cnn_h, d.cnn_w, d.cnn_k, d.cnn_cout, d.cnn_hidden, d.cnn_classes) = cnn
        for i, v in enumerate(fwd_frac_bits or []):   # per-layer forward-weight bits (R21)
            d.fwd_frac_bits[i] = v
        d.compare = compare                           # 0 A2B chain (R9), 1 FSS comparison (R22)
        d.weight_decay_shift = weight_decay_shift     # SVM weight decay (R24)
        d.rnn_steps = rnn_steps                       # RNN sequence length (R25)
        d.deal_role = deal_role                       # 0 dealer, 1/2 party 0/1 dealing for itself (R23)
        d.mask_reuse = 1 if mask_reuse else 0         # forward/backward mask reuse (R26)
        d.strong_pairs = strong_pairs                 # strong-scaling dealer layout
        self.ctx, self.desc, self.kind = ctx, d, kind
        h = vp()
        _call("psml_model_create", ctx.handle, ctypes.byref(d), ctypes.byref(h))
        self.handle = h
        self.n_layers = d.n_layers
        # words per minibatch of one party's input / label shares (guards the ABI calls)
        x_row = (cnn[0] * cnn[1] * cnn[2] if kind == CNN else
                 (rnn_steps * dims[0] if kind == RNN else dims[0]))
        self.x_words = batch * x_row
        self.y_words = batch * self.layer_shape(self.n_layers - 1)[1]
        self.ring_dtypes = (dtype_of(ctx.l), torch.int64 if ctx.l == 64 else torch.int32)

    def layer_shape(self, layer):
        r, c = i64(), i64()
        _call("psml_model_layer_shape", self.handle, layer, ctypes.byref(r), ctypes.byref(c))
        return r.value, c.value

    def set_master(self, layer, Wm, stream=None):
        _call("psml_model_set_master", self.handle, layer, _pair(Wm), _stream(stream))

    def get_master(self, layer, stream=None):
        W = empty_pair(self.layer_shape(layer), self.ctx.l)
        _call("psml_model_get_master", self.handle, layer, _pair(W), _stream(stream))
        return W

    def deal(self, step, infer_only=False, stream=None):
        _call("psml_model_deal", self.handle, step, 1 if infer_only else 0, _stream(stream))

    def deal_bundle(self, step, party, stream=None):
        """Dealer side (deal_role 0): deal `step` and return party `party`'s derived words (R23)."""
        w = i64()
        _call("psml_model_deal_bundle", self.handle, step, party, None, ctypes.byref(w), _stream(stream))
        b = torch.empty(max(w.value, 1), dtype=dtype_of(self.ctx.l), device="cuda")
        _call("psml_model_deal_bundle", self.handle, step, party, _ptr(b), ctypes.byref(w), _stream(stream))
        return b[:w.value]

    def deal_party(self, step, party, bundle=None, stream=None):
        """Party side (deal_role party + 1): own streams + the dealer's bundle (R23)."""
        n = 0 if bundle is None else bundle.numel()
        _call("psml_model_deal_party", self.handle, step, party, _ptr(bundle) if n else None, n, _stream(stream))

    def _xy(self, X, Y):
        _check(X, self.x_words, self.ring_dtypes, "X shares")
        _check(Y, self.y_words, self.ring_dtypes, "Y shares")

    def train_step(self, X, Y, step, stream=None):
        self._xy(X, Y)
        _call("psml_secure_train_step", self.handle, _pair(X), _pair(Y), step, _stream(stream))

    def forward_backward(self, X, Y, step, stream=None):
        self._xy(X, Y)
        _call("psml_train_forward_backward", self.handle, _pair(X), _pair(Y), step,
              _stream(stream))

    def output(self):
        """Model-owned prediction shares (ptr0, ptr1, words) of the last forward pass."""
        a, b, n = vp(), vp(), i64()
        _call("psml_model_output", self.handle, ctypes.byref(a), ctypes.byref(b), ctypes.byref(n))
        return a.value, b.value, n.value

    def grads(self):
        """(pointer, words per party) of the model-owned [2][P] gradient buffer."""
        p, n = vp(), i64()
        _call("psml_model_grads", self.handle, ctypes.byref(p), ctypes.byref(n))
        return p.value, n.value

    def apply_update(self, extra_shift=0, stream=None):
        _call("psml_train_apply_update", self.handle, extra_shift, _stream(stream))

    def capture_step(self, X, Y, with_deal=True, with_update=True, pipelined=False, stream=None,
                     unsafe_reuse_material=False):
        """Capture one step into a CUDA graph reading the fixed share buffers X, Y (pipelined:
        the dealer of step s + 1 overlaps the online phase of step s).  unsafe_reuse_material
        (benchmark-only timing of the online phase): replay the material dealt once into pool 0
        on every step -- never in a real run, reused masks leak."""
        self._xy(X, Y)
        flags = ((1 if with_deal else 0) | (2 if with_update else 0) | (4 if pipelined else 0)
                 | (8 if unsafe_reuse_material else 0))
        _call("psml_model_capture_step", self.handle, _pair(X), _pair(Y), flags, _stream(stream))

    def graph_nodes(self):
        n = i64()
        _call("psml_model_graph_nodes", self.handle, ctypes.byref(n))
        return n.value

    def step_graph(self, step, stream=None):
        _call("psml_model_step_graph", self.handle, step, _stream(stream))

    def step_device(self, X, Y, share_seed, step, stream=None):
        """psml_model_step_device: X, Y float64 device tensors (the batch in HBM); one launch
        encodes and shares both into the captured buffers, then the captured step replays."""
        _check(X, self.x_words, (torch.float64,), "step_device X")
        _check(Y, self.y_words, (torch.float64,), "step_device Y")
        _call("psml_model_step_device", self.handle, _ptr(X), _ptr(Y), share_seed, step, _stream(stream))

    def step_host(self, q, y, share_seed, step, yhat_host, stream=None):
        """psml_model_step_host: q uint8 pixels, y float64 labels or uint8 class indices, yhat_host
        a (2, batch, d_L) uint64 CPU tensor -- all host tensors (pinned)."""
        if q.dtype != torch.uint8 or y.dtype not in (torch.uint8, torch.float64) or yhat_host.dtype != torch.uint64:
            raise PsmlError("marshal", 1, "step_host: q uint8, y float64 | uint8, yhat_host uint64")
        batch = self.desc.batch
        want_y = batch if y.dtype == torch.uint8 else self.y_words
        if q.numel() != self.x_words or y.numel() != want_y or yhat_host.numel() < 2 * self.y_words:
            raise PsmlError("marshal", 2, f"step_host: q {q.numel()} (want {self.x_words}), y {y.numel()} "
                                          f"(want {want_y}), yhat_host {yhat_host.numel()} (want >= {2 * self.y_words})")
        _call("psml_model_step_host", self.handle, _host_ptr(q), _host_ptr(y), 1 if y.dtype == torch.uint8 else 0,
              share_seed, step, _host_ptr(yhat_host), _stream(stream))

    def party_train_step(self, party, xport, dp, X_i, Y_i, step, stream=None):
        """Split deployment: forward/backward + this party's gradient all-reduce over `dp`
        (DataParallel or None) + update (psml_party_train_step)."""
        self._xy(X_i, Y_i)
        _call("psml_party_train_step", self.handle, party, xport.handle, dp.handle if dp else None,
              _ptr(X_i), _ptr(Y_i), step, _stream(stream))

    def party_capture_step(self, party, xport, dp, X_i, Y_i, with_deal=True, with_update=True,
                           pipelined=False, stream=None):
        self._xy(X_i, Y_i)
        flags = (1 if with_deal else 0) | (2 if with_update else 0) | (4 if pipelined else 0)
        _call("psml_party_capture_step", self.handle, party, xport.handle, dp.handle if dp else None,
              _ptr(X_i), _ptr(Y_i), flags, _stream(stream))

    def party_forward_backward(self, party, xport, X_i, Y_i, step, stream=None):
        """Split deployment: party `party`'s half of the step, openings through `xport`."""
        self._xy(X_i, Y_i)
        _call("psml_party_forward_backward", self.handle, party, xport.handle, _ptr(X_i), _ptr(Y_i),
              step, _stream(stream))

    def party_apply_update(self, party, extra_shift=0, stream=None):
        _call("psml_party_apply_update", self.handle, party, extra_shift, _stream(stream))

    def infer(self, X, step, out_shape, stream=None):
        _check(X, self.x_words, self.ring_dtypes, "X shares")
        Y = empty_pair(out_shape, self.ctx.l)
        _check(Y, self.y_words, self.ring_dtypes, "prediction buffers")
        _call("psml_secure_infer", self.handle, _pair(X), step, _pair(Y), _stream(stream))
        return Y

    def close(self):
        if self.handle:
            lib().psml_model_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


# ---------------------------------------------------------------------------------------------
# split-deployment transports
# ---------------------------------------------------------------------------------------------
def nccl_unique_id():
    buf = (ctypes.c_uint8 * 128)()
    _call("psml_nccl_unique_id", ctypes.cast(buf, vp))
    return bytes(buf)


class Transport:
    """psml_xport: how a party's masked messages reach its peer (include/psml.h)."""

    def __init__(self, handle, keep=None):
        self.handle = handle
        self._keep = keep   # the ctypes callback must outlive the transport

    @classmethod
    def nccl(cls, uid, rank):
        """Library-owned 2-rank NCCL communicator (this party = rank) on the current device."""
        buf = (ctypes.c_uint8 * 128).from_buffer_copy(uid)
        h = vp()
        _call("psml_xport_nccl_create", ctypes.cast(buf, vp), rank, ctypes.byref(h))
        return cls(h)

    @classmethod
    def callback(cls, fn):
        """fn(msgs, stream_ptr): msgs = [(send_ptr, recv_ptr, nbytes)]; must deliver each send
        buffer to the peer and fill each recv buffer, ordered on the stream."""
        def tramp(_user, n, send, recv, nbytes, stream):
            try:
                fn([(send[k], recv[k], nbytes[k]) for k in range(n)], stream)
                return 0
            except Exception as e:   # noqa: BLE001 -- reported through the status code
                import sys
                print(f"psml exchange callback failed: {e!r}", file=sys.stderr)
                return 1
        cb = EXCHANGE_FN(tramp)
        h = vp()
        _call("psml_xport_callback_create", cb, None, ctypes.byref(h))
        return cls(h, keep=cb)

    @classmethod
    def peer(cls, party, capacity_bytes=64 << 20):
        """Peer-memory transport (psml_xport_peer_create): returns (transport, handle blob); ship
        the blob to the peer and call connect() with the peer's blob."""
        buf = (ctypes.c_uint8 * PEER_HANDLE_BYTES)()
        h = vp()
        _call("psml_xport_peer_create", party, capacity_bytes, ctypes.byref(h), ctypes.cast(buf, vp))
        return cls(h), bytes(buf)

    def connect(self, peer_handle):
        buf = (ctypes.c_uint8 * PEER_HANDLE_BYTES).from_buffer_copy(peer_handle)
        _call("psml_xport_peer_connect", self.handle, ctypes.cast(buf, vp))

    def stats(self):
        b, n = i64(), i64()
        _call("psml_xport_stats", self.handle, ctypes.byref(b), ctypes.byref(n))
        return b.value, n.value

    def close(self):
        if self.handle:
            lib().psml_xport_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class DataParallel:
    """psml_dp: one party's library-owned NCCL communicator over its data-parallel GPUs."""

    def __init__(self, uid, rank, size):
        h = vp()
        if uid is None:
            _call("psml_dp_create", None, rank, size, ctypes.byref(h))
        else:
            buf = (ctypes.c_uint8 * 128).from_buffer_copy(uid)
            _call("psml_dp_create", ctypes.cast(buf, vp), rank, size, ctypes.byref(h))
        self.handle = h
        self.size = size

    def allreduce_(self, t, stream=None):
        """In-place Z_{2^l} sum of a contiguous uint64 / uint32 CUDA tensor over the group."""
        l = 64 if t.dtype in (torch.uint64, torch.int64) else 32
        _call("psml_dp_allreduce", self.handle, _ptr(t), t.numel(), l, _stream(stream))
        return t

    def close(self):
        if self.handle:
            lib().psml_dp_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def wrap_bytes(ptr, nbytes):
    """A uint8 torch tensor aliasing `nbytes` bytes of device memory at `ptr`."""
    class _Holder:
        __cuda_array_interface__ = {"shape": (nbytes,), "typestr": "|u1", "data": (ptr, False),
                                    "version": 3, "strides": None}
    return torch.as_tensor(_Holder(), device="cuda")
