"""ctypes marshalling of oracle/psml_oracle.c, plus the plain numpy pieces of the protocol.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).  All ring values are numpy uint64 arrays
holding residues mod 2^l (for l < 64 the high bits are zero).  Both parties are simulated.
"""
import ctypes
import numpy as np

from . import build

_lib = None
U64P = ctypes.POINTER(ctypes.c_uint64)


def lib():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        L = _lib
        c_i, c_i64, c_u64, c_u32, vp = (ctypes.c_int, ctypes.c_int64, ctypes.c_uint64,
                                        ctypes.c_uint32, ctypes.c_void_p)
        L.or_chacha20_block.argtypes = [vp, c_u32, vp, vp]
        L.or_prg.argtypes = [c_i, c_u64, c_u32, c_u64, c_u64, c_i64, vp]
        L.or_encode.argtypes = [c_i, c_i, vp, c_i64, vp]
        L.or_decode.argtypes = [c_i, c_i, vp, c_i64, vp]
        L.or_share.argtypes = [c_i, c_u64, c_u64, vp, c_i64, vp, vp]
        L.or_reconstruct.argtypes = [c_i, vp, vp, c_i64, vp]
        L.or_ring_matmul.argtypes = [c_i, vp, vp, c_i64, c_i64, c_i64, vp]
        L.or_triplet_gen.argtypes = [c_i, c_u64, c_u64, c_i64, c_i64, c_i64] + [vp] * 6
        L.or_hadamard_triplet_gen.argtypes = [c_i, c_u64, c_u64, c_i64] + [vp] * 6
        L.or_beaver_matmul.argtypes = ([c_i, c_i] + [vp] * 10 + [c_i64, c_i64, c_i64, c_i]
                                       + [vp] * 8)
        L.or_beaver_hadamard.argtypes = [c_i] + [vp] * 10 + [c_i64, vp, vp]
        L.or_truncate.argtypes = [c_i, c_i, vp, c_i64, c_i]
        L.or_msb_material_words.argtypes = [c_i, c_i64]
        L.or_msb_material_words.restype = c_i64
        L.or_msb_dealer.argtypes = [c_i, c_u64, c_u64, c_i64, vp, vp]
        L.or_secure_msb.argtypes = [c_i, vp, vp, c_i64, vp, vp, vp, vp, vp, vp]
        L.or_delta_csr_encode.argtypes = [c_i, vp, vp, c_i64, c_i64, vp, vp, vp, vp, vp]
        L.or_delta_csr_encode.restype = c_i64
        L.or_delta_csr_apply.argtypes = [c_i, c_i64, c_i64, ctypes.c_int32, vp, vp, vp, vp, vp]
        L.or_num_threads.restype = c_i
        L.or_party_seed.argtypes = [c_u64, c_i]
        L.or_party_seed.restype = c_u64
        L.or_stream_seed.argtypes = [c_u64, c_u32]
        L.or_stream_seed.restype = c_u64
        L.or_dcf_key_words.argtypes = [c_i]
        L.or_dcf_key_words.restype = c_i64
        L.or_dcf_gen.argtypes = [c_i, c_i, c_u64, c_u64, c_u64, c_u64, c_u64, c_u64, vp, vp]
        L.or_dcf_eval.argtypes = [c_i, c_i, c_i, vp, c_u64]
        L.or_dcf_eval.restype = c_u64
        L.or_fss_words.argtypes = [c_i]
        L.or_fss_words.restype = c_i64
        L.or_fss_dealer.argtypes = [c_i, c_u64, c_u64, c_i64, vp, vp]
        L.or_fss_drelu.argtypes = [c_i, vp, vp, c_i64, vp, vp, vp, vp, vp]
    return _lib


def _p(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _u64(a):
    a = np.ascontiguousarray(a, dtype=np.uint64)
    return a


def mask(l):
    return np.uint64((1 << l) - 1) if l < 64 else np.uint64(0xFFFFFFFFFFFFFFFF)


def tag(s: str) -> int:
    """4-byte role tag (R1), little-endian packing of up to 4 bytes."""
    b = s.encode() if isinstance(s, str) else bytes(s)
    b = (b + b"\0\0\0\0")[:4]
    return int.from_bytes(b, "little")


def num_threads():
    return lib().or_num_threads()


# ---------------------------------------------------------------------------------------------
# PRG (ChaCha20 counter mode, R1)
# ---------------------------------------------------------------------------------------------
def chacha20_block(key_words, counter, nonce_words):
    k = np.ascontiguousarray(key_words, dtype=np.uint32)
    n = np.ascontiguousarray(nonce_words, dtype=np.uint32)
    out = np.zeros(16, dtype=np.uint32)
    lib().or_chacha20_block(_p(k), counter, _p(n), _p(out))
    return out


def party_seed(dealer_seed, party):
    """s_i = PRG(dealer_seed, "KD", i)[0] (R23)."""
    return lib().or_party_seed(dealer_seed, party)


def stream_seed(dealer_seed, tag_value):
    """The seed a dealer material stream is keyed by (R23): the owning party's, or the dealer's."""
    return lib().or_stream_seed(dealer_seed, tag_value)


def dealer_prg(l, dealer_seed, tag_value, call_id, n, offset=0):
    return prg(l, stream_seed(dealer_seed, tag_value), tag_value, call_id, n, offset)


def prg(l, seed, tag_value, call_id, n, offset=0):
    out = np.empty(n, dtype=np.uint64)
    lib().or_prg(l, seed, tag_value, call_id, offset, n, _p(out))
    return out


# ---------------------------------------------------------------------------------------------
# encode / share / reconstruct
# ---------------------------------------------------------------------------------------------
def encode(x, l=64, f=13):
    x = np.ascontiguousarray(x, dtype=np.float64)
    v = np.empty(x.shape, dtype=np.uint64)
    lib().or_encode(l, f, _p(x), x.size, _p(v))
    return v


def decode(v, l=64, f=13):
    v = _u64(v)
    x = np.empty(v.shape, dtype=np.float64)
    lib().or_decode(l, f, _p(v), v.size, _p(x))
    return x


def share(x, seed, stream, l=64):
    x = _u64(x)
    x0 = np.empty_like(x)
    x1 = np.empty_like(x)
    lib().or_share(l, seed, stream, _p(x), x.size, _p(x0), _p(x1))
    return x0, x1


def reconstruct(x0, x1, l=64):
    x0, x1 = _u64(x0), _u64(x1)
    x = np.empty_like(x0)
    lib().or_reconstruct(l, _p(x0), _p(x1), x0.size, _p(x))
    return x


def ring_matmul(A, B, l=64):
    A, B = _u64(A), _u64(B)
    M, K = A.shape
    K2, N = B.shape
    assert K == K2
    C = np.empty((M, N), dtype=np.uint64)
    lib().or_ring_matmul(l, _p(A), _p(B), M, K, N, _p(C))
    return C


def truncate(x, party, d, l=64):
    y = _u64(x).copy()
    lib().or_truncate(l, party, _p(y), y.size, d)
    return y


# ---------------------------------------------------------------------------------------------
# dealer
# ---------------------------------------------------------------------------------------------
def triplet_gen(seed, call_id, M, K, N, l=64):
    """Returns (U0, U1, V0, V1, Z0, Z1); U: MxK, V: KxN, Z: MxN (Eqs. 2-3)."""
    U0, U1 = np.empty((M, K), np.uint64), np.empty((M, K), np.uint64)
    V0, V1 = np.empty((K, N), np.uint64), np.empty((K, N), np.uint64)
    Z0, Z1 = np.empty((M, N), np.uint64), np.empty((M, N), np.uint64)
    lib().or_triplet_gen(l, seed, call_id, M, K, N, *map(_p, (U0, U1, V0, V1, Z0, Z1)))
    return U0, U1, V0, V1, Z0, Z1


def hadamard_triplet_gen(seed, call_id, n, l=64):
    arrs = [np.empty(n, np.uint64) for _ in range(6)]
    lib().or_hadamard_triplet_gen(l, seed, call_id, n, *map(_p, arrs))
    return tuple(arrs)


def msb_dealer(seed, call_id, n, l=64):
    w = lib().or_msb_material_words(l, n)
    m0, m1 = np.empty(w, np.uint64), np.empty(w, np.uint64)
    lib().or_msb_dealer(l, seed, call_id, n, _p(m0), _p(m1))
    return m0, m1


# ---------------------------------------------------------------------------------------------
# online protocol pieces
# ---------------------------------------------------------------------------------------------
def beaver_matmul(A, B, trip, trunc=0, form=0, l=64, trace=False):
    """Both parties' Beaver product shares (Eqs. 4-6; form 0 = BJ canonical)."""
    (A0, A1), (B0, B1) = [tuple(map(_u64, t)) for t in (A, B)]
    U0, U1, V0, V1, Z0, Z1 = map(_u64, trip)
    M, K = A0.shape
    N = B0.shape[1]
    C0, C1 = np.empty((M, N), np.uint64), np.empty((M, N), np.uint64)
    tr = ([np.empty((M, K), np.uint64) for _ in range(3)]
          + [np.empty((K, N), np.uint64) for _ in range(3)]) if trace else [None] * 6
    lib().or_beaver_matmul(l, form, *map(_p, (A0, A1, B0, B1, U0, U1, V0, V1, Z0, Z1)),
                           M, K, N, trunc, _p(C0), _p(C1), *map(_p, tr))
    if trace:
        return (C0, C1), dict(E0=tr[0], E1=tr[1], E=tr[2], F0=tr[3], F1=tr[4], F=tr[5])
    return C0, C1


def beaver_hadamard(A, B, trip, l=64):
    (A0, A1), (B0, B1) = [tuple(map(_u64, t)) for t in (A, B)]
    shape = A0.shape
    args = [a.reshape(-1) for a in (A0, A1, B0, B1)] + [_u64(t).reshape(-1) for t in trip]
    n = A0.size
    C0, C1 = np.empty(n, np.uint64), np.empty(n, np.uint64)
    lib().or_beaver_hadamard(l, *map(_p, args), n, _p(C0), _p(C1))
    return C0.reshape(shape), C1.reshape(shape)


def secure_msb(x, mat, l=64, want_bool=False):
    """Arithmetic shares of MSB(x_0 + x_1) via Kogge-Stone A2B + daBit B2A (R9)."""
    x0, x1 = _u64(x[0]).reshape(-1), _u64(x[1]).reshape(-1)
    n = x0.size
    outs = [np.empty(n, np.uint64) for _ in range(4)]
    lib().or_secure_msb(l, _p(x0), _p(x1), n, _p(mat[0]), _p(mat[1]), *map(_p, outs))
    shape = np.shape(x[0])
    if want_bool:
        return ((outs[0].reshape(shape), outs[1].reshape(shape)),
                (outs[2].reshape(shape), outs[3].reshape(shape)))
    return outs[0].reshape(shape), outs[1].reshape(shape)


def secure_relu(x, mat, htrip, l=64):
    """ReLU(x) = x (.) (1 - msb(x)) (Beaver Hadamard); returns (relu shares, drelu shares)."""
    m = mask(l)
    msb0, msb1 = secure_msb(x, mat, l)
    d0 = (np.uint64(1) - msb0) & m          # public constant 1 added by party 0 only
    d1 = (np.uint64(0) - msb1) & m
    r0, r1 = beaver_hadamard(x, (d0, d1), htrip, l)
    return (r0, r1), (d0, d1)


def eq9_inputs(z, l=64, f=13):
    """[z + 1/2 ; z - 1/2] with the public constant added by party 0 only (Eq. 9)."""
    m = mask(l)
    h = np.uint64(1 << (f - 1))
    z0, z1 = _u64(z[0]).reshape(-1), _u64(z[1]).reshape(-1)
    x0 = np.concatenate([(z0 + h) & m, (z0 - h) & m])
    return x0, np.concatenate([z1, z1])


def secure_eq9(z, mat, htrip, l=64, f=13):
    """Eq. 9 f(x) = ReLU(x + 1/2) - ReLU(x - 1/2) (= clamp(x + 1/2, 0, 1), R8)."""
    m = mask(l)
    n = np.size(z[0])
    x = eq9_inputs(z, l, f)
    (r0, r1), _ = secure_relu(x, mat, htrip, l)
    shape = np.shape(z[0])
    y0 = ((r0[:n] - r0[n:]) & m).reshape(shape)
    y1 = ((r1[:n] - r1[n:]) & m).reshape(shape)
    return y0, y1


# ---------------------------------------------------------------------------------------------
# one-round secure comparison by FSS (DCF, R22)
# ---------------------------------------------------------------------------------------------
def dcf_gen(l, n_bits, alpha, beta, seed0, seed1):
    """DCF keys of f(x) = beta * [x < alpha] on n_bits inputs; seeds are (lo, hi) 128-bit pairs."""
    kw = lib().or_dcf_key_words(n_bits)
    k0, k1 = np.empty(kw, np.uint64), np.empty(kw, np.uint64)
    lib().or_dcf_gen(l, n_bits, alpha, beta, seed0[0], seed0[1], seed1[0], seed1[1], _p(k0), _p(k1))
    return k0, k1


def dcf_eval(l, n_bits, b, key, x):
    return lib().or_dcf_eval(l, n_bits, b, _p(_u64(key)), int(x))


def fss_dealer(seed, call_id, n, l=64):
    w = lib().or_fss_words(l) * n
    m0, m1 = np.empty(w, np.uint64), np.empty(w, np.uint64)
    lib().or_fss_dealer(l, seed, call_id, n, _p(m0), _p(m1))
    return m0, m1


def fss_drelu(x, mat, l=64, trace=False):
    """Arithmetic shares of DReLU(x) = [x >= 0] after ONE opening (xhat = x + r) + DCF evaluation."""
    x0, x1 = _u64(x[0]).reshape(-1), _u64(x[1]).reshape(-1)
    n = x0.size
    d0, d1, xh = np.empty(n, np.uint64), np.empty(n, np.uint64), np.empty(n, np.uint64)
    lib().or_fss_drelu(l, _p(x0), _p(x1), n, _p(mat[0]), _p(mat[1]), _p(d0), _p(d1), _p(xh))
    shape = np.shape(x[0])
    out = (d0.reshape(shape), d1.reshape(shape))
    return (out, xh.reshape(shape)) if trace else out


def secure_relu_fss(x, mat, htrip, l=64):
    """ReLU(x) = x (.) DReLU(x): the FSS comparison round, then one Beaver Hadamard round."""
    d = fss_drelu(x, mat, l)
    r = beaver_hadamard((_u64(x[0]).reshape(-1), _u64(x[1]).reshape(-1)),
                        (d[0].reshape(-1), d[1].reshape(-1)), htrip, l)
    shape = np.shape(x[0])
    return (r[0].reshape(shape), r[1].reshape(shape)), d


# ---------------------------------------------------------------------------------------------
# CSR delta codec
# ---------------------------------------------------------------------------------------------
def delta_csr_encode(cur, prev, l=64):
    cur, prev = _u64(cur), _u64(prev)
    rows, cols = cur.shape
    is_csr = np.zeros(1, np.int32)
    row_ptr = np.zeros(rows + 1, np.int32)
    col_idx = np.zeros(rows * cols, np.int32)
    vals = np.zeros(rows * cols, np.uint64)
    dense = np.zeros(rows * cols, np.uint64)
    nnz = lib().or_delta_csr_encode(l, _p(cur), _p(prev), rows, cols, _p(is_csr), _p(row_ptr),
                                    _p(col_idx), _p(vals), _p(dense))
    if is_csr[0]:
        return dict(is_csr=True, nnz=nnz, row_ptr=row_ptr, col_idx=col_idx[:nnz], vals=vals[:nnz])
    return dict(is_csr=False, nnz=nnz, dense=dense.reshape(rows, cols))


def delta_csr_apply(target, enc, l=64):
    t = _u64(target).copy()
    rows, cols = t.shape
    if enc["is_csr"]:
        lib().or_delta_csr_apply(l, rows, cols, 1, _p(enc["row_ptr"]), _p(enc["col_idx"]),
                                 _p(_u64(enc["vals"])), None, _p(t))
    else:
        lib().or_delta_csr_apply(l, rows, cols, 0, None, None, None,
                                 _p(_u64(enc["dense"]).reshape(-1)), _p(t))
    return t


# ---------------------------------------------------------------------------------------------
# im2col (CNN row of SURVEY 8(a) a6; R17): rows (b, oy, ox), cols (c, ky, kx)
# ---------------------------------------------------------------------------------------------
def im2col(X, C, H, W, k):
    """X: (B, C*H*W) -> (B*OH*OW, C*k*k), valid padding, stride 1.  Pure indexing."""
    B = X.shape[0]
    OH, OW = H - k + 1, W - k + 1
    X4 = X.reshape(B, C, H, W)
    out = np.empty((B, OH, OW, C, k, k), dtype=X.dtype)
    for ky in range(k):
        for kx in range(k):
            out[:, :, :, :, ky, kx] = X4[:, :, ky:ky + OH, kx:kx + OW].transpose(0, 2, 3, 1)
    return out.reshape(B * OH * OW, C * k * k)
