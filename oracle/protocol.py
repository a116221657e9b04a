"""Secure training / inference protocols, both parties simulated -- TEST INFRASTRUCTURE ONLY.

Follows PAPER.md Sec. 4.3 "Detailed Design" (L201-L207): each layer runs a forward
reconstruct (masking + opening) and a forward operation (Eq. 6/8), then a backward reconstruct
and backward operation; B_i is the model, updated every step.  The fixed-point, truncation,
activation-protocol, learning-rate and master-weight readings are DESIGN.md R3, R7, R9, R10,
R13-R17.  The call-id layout (R11) is part of the parity contract with the CUDA path:

    call_id = pair[63:56] | step[55:24] | layer[23:16] | op[15:8] | slot[7:0]

ops: 0 forward matmul, 1 weight gradient, 2 input gradient, 3 ReLU MSB, 4 Eq. 9 MSB,
6 Hadamard (slot 0 ReLU, 1 backprop DReLU, 2 Eq. 9), 7 share (slot 0 X, 1 Y, 2 init weight).

All values are uint64 numpy arrays in Z_{2^64} (training is l = 64 only, R18).
"""
import numpy as np

from . import core

DATA_SEED = 0x50534D4C
SHARE_SEED = DATA_SEED + 1
DEALER_SEED = DATA_SEED + 2

OP_FWD, OP_GRADW, OP_GRADIN, OP_RELU_MSB, OP_EQ9_MSB, OP_B2A, OP_HADAMARD, OP_SHARE = range(8)
INIT_STEP = 0xFFFFFFFF

F = 13            # fractional bits of activations / data / forward weights
LR_SHIFT = 14     # eta / |B| = 2^-14  (eta = 2^-7, |B| = 128)
MASTER = 27       # master-weight fractional bits m = F + LR_SHIFT (R14)
L = 64
MASK = np.uint64(0xFFFFFFFFFFFFFFFF)

CNN_GEOM = dict(C=3, H=32, W=32, k=5, Cout=16, hidden=64, classes=10)

# Forward-weight precision f_w per layer (R21).  The forward copy of a layer's weights
# keeps f_w fractional bits, W = trunc(W^m, MASTER - f_w), and every product with it (forward
# h.W and backprop delta.W^T) is truncated by f_w, so activations and deltas stay at F = 13 bits.
# f_w = F except the CNN, whose 12544-wide FC1 and 5x5 conv fail BJ's 2^-12 weight bound at
# f_w = 13 (weights of magnitude ~0.005 quantised at 2^-13 perturb every pre-activation).
FWD_BITS = {"linreg": [F], "logreg": [F], "svm": [F], "mlp": [F, F, F], "cnn": [16, 20, 20], "rnn": [F, F]}
RNN_GEOM = dict(T=16, D=32, H=64, C=10)   # DESIGN.md R25 (synth.RNN_*)
# linear SVM (R24): weight decay lambda.eta = 2^-WD_SHIFT applied to the master weights
WD_SHIFT = 16


def call_id(pair, step, layer, op, slot=0):
    return ((pair & 0xFF) << 56) | ((step & 0xFFFFFFFF) << 24) | ((layer & 0xFF) << 16) \
        | ((op & 0xFF) << 8) | (slot & 0xFF)


def dims_of(task):
    return {"linreg": [784, 1], "logreg": [784, 1], "svm": [784, 1], "mlp": [784, 128, 128, 10],
            "cnn": [None, 12544, 64, 10]}[task]


# ---------------------------------------------------------------------------------------------
# client side: encode + share
# ---------------------------------------------------------------------------------------------
def share_batch(X, Y, step, pair=0):
    x = core.encode(X, L, F)
    y = core.encode(Y, L, F)
    pf = _field(pair)   # strong scaling: each pair's client shares its own rows afresh
    return (core.share(x, SHARE_SEED, call_id(pf, step, 0, OP_SHARE, 0)),
            core.share(y, SHARE_SEED, call_id(pf, step, 0, OP_SHARE, 1)))


def trunc_pair(x, d):
    return core.truncate(x[0], 0, d), core.truncate(x[1], 1, d)


# ---------------------------------------------------------------------------------------------
# Diagnostics: the oracle knows the plaintext, so it counts SecureML
# truncation failures (|t - floor(x / 2^d)| > 1, R7: probability <= 2^(l_x + 1 - l) each) and
# secure-comparison mismatches (DReLU != [x >= 0], Eq. 9 output != clamp(x + 1/2, 0, 1), R8/R9).
# A fixed-seed run must report 0 of each.  Off by default (costs a reconstruction per check).
# ---------------------------------------------------------------------------------------------
DIAG = {"on": False, "trunc_checked": 0, "trunc_fail": 0, "msb_checked": 0, "msb_fail": 0}


def diag_reset(on=True):
    DIAG.update(on=on, trunc_checked=0, trunc_fail=0, msb_checked=0, msb_fail=0)


def _signed(v):
    return np.asarray(v, dtype=np.uint64).view(np.int64)


def check_trunc(pre, post, d):
    """Count elements whose truncated reconstruction is more than 1 LSB from floor(x / 2^d)."""
    if not DIAG["on"] or d == 0:
        return
    x = _signed(pre[0] + pre[1])
    t = _signed(post[0] + post[1])
    diff = t - (x >> np.int64(d))          # int64 wraparound keeps a failure far outside [-1, 1]
    DIAG["trunc_checked"] += int(x.size)
    DIAG["trunc_fail"] += int(np.count_nonzero((diff > 1) | (diff < -1)))


def checked_trunc(x, d):
    t = trunc_pair(x, d)
    check_trunc(x, t, d)
    return t


def sub_pair(a, b):
    return a[0] - b[0], a[1] - b[1]


class Model:
    """Both parties' weight shares: master (MASTER fractional bits) and forward copy (fw[l] bits)."""

    def __init__(self, task, W_init, fw=None, compare="a2b", mask_reuse=False):
        self.task = task
        self.mask_reuse = mask_reuse   # SecureML forward/backward mask reuse (R26; MLP family only)
        assert not mask_reuse or task in ("linreg", "logreg", "mlp")
        self.compare = compare   # secure comparison of ReLU / Eq. 9: "a2b" (R9) or "fss" (R22)
        self.fw = list(fw) if fw is not None else list(FWD_BITS[task])
        if task == "mlp" and fw is None:
            self.fw = [F] * len(W_init)
        assert len(self.fw) == len(W_init)
        self.Wm = []
        for layer, W in enumerate(W_init):
            w = core.encode(W, L, MASTER)
            self.Wm.append(core.share(w, SHARE_SEED, call_id(0, INIT_STEP, layer, OP_SHARE, 2)))
        self.W = [trunc_pair(wm, MASTER - f) for wm, f in zip(self.Wm, self.fw)]

    def decoded_master(self):
        return [core.decode(core.reconstruct(*wm), L, MASTER) for wm in self.Wm]


# ---------------------------------------------------------------------------------------------
# dealer-aided building blocks (both parties)
# ---------------------------------------------------------------------------------------------
def _T(p):
    return np.ascontiguousarray(p[0].T), np.ascontiguousarray(p[1].T)


class Strong:
    """Pair k of P under strong scaling (R28): the P pairs train on ONE
    global batch of P b rows, pair k on rows [k b, (k + 1) b).  Every op whose output rows are
    batch rows -- forward and input-gradient products, ReLU / Eq. 9, Hadamard -- takes the
    row-slices of the material a single pair would draw for the whole global batch (pair field 0;
    the weight mask V is the global one, shared: every pair opens the same F = W - V of the same
    replicated W).  Weight-gradient products contract over the batch and take independent
    per-pair triplets (pair field k).  A mask is never reused on two different values."""

    def __init__(self, k, P):
        assert 0 <= k < P
        self.k, self.P = k, P


def _field(pair):
    """Call-id pair field of a pair's own (per-pair) material."""
    return pair.k if isinstance(pair, Strong) else pair


def _slice_idx(pair, n, parts):
    """Global element indices of pair k's n elements: `parts` row-ordered blocks of n / parts
    (Eq. 9's [z + 1/2 ; z - 1/2]), block h of the global layout holding P n / parts elements."""
    per = n // parts
    return np.concatenate([h * pair.P * per + pair.k * per + np.arange(per) for h in range(parts)])


def mat_triplet(pair, step, layer, op, M, K, N):
    """Matrix triplet of the product (layer, op) with M output rows."""
    if isinstance(pair, Strong) and op != OP_GRADW:
        U0, U1, V0, V1, Z0, Z1 = core.triplet_gen(DEALER_SEED, call_id(0, step, layer, op, 0), pair.P * M, K, N, L)
        r = slice(pair.k * M, (pair.k + 1) * M)
        return U0[r], U1[r], V0, V1, Z0[r], Z1[r]
    return core.triplet_gen(DEALER_SEED, call_id(_field(pair), step, layer, op, 0), M, K, N, L)


def had_triplet(pair, step, layer, slot, n, parts=1):
    if isinstance(pair, Strong):
        t = core.hadamard_triplet_gen(DEALER_SEED, call_id(0, step, layer, OP_HADAMARD, slot), pair.P * n, L)
        i = _slice_idx(pair, n, parts)
        return tuple(a[i] for a in t)
    return core.hadamard_triplet_gen(DEALER_SEED, call_id(pair, step, layer, OP_HADAMARD, slot), n, L)


def cmp_material(pair, step, layer, op, n, compare, parts=1):
    """Comparison material of n elements: A2B chain (R9, 11 planes of n words) or DCF keys (R22,
    257 planes); plane-major, so a pair's slice is the same element range of every plane."""
    gen = core.fss_dealer if compare == "fss" else core.msb_dealer
    if isinstance(pair, Strong):
        ng = pair.P * n
        i = _slice_idx(pair, n, parts)
        return tuple(np.ascontiguousarray(m.reshape(-1, ng)[:, i]).reshape(-1)
                     for m in gen(DEALER_SEED, call_id(0, step, layer, op, 0), ng, L))
    return gen(DEALER_SEED, call_id(pair, step, layer, op, 0), n, L)


def reuse_triplets(pair, step, layer, B, din, dout):
    """SecureML forward/backward mask reuse (R26): the backward
    products of layer l re-use the masks of values already opened -- the activation A_l's forward
    mask U_f (gradW's left operand A_l^T - U_f^T = E_f^T) and the weight's forward mask V_f (gradin's
    right operand W_l^T - V_f^T = F_f^T) -- and ONE fresh mask D of delta serves both products
    (gradW's right operand and gradin's left operand).  D_i = PRG("U0"/"U1") and Z_0 = PRG("Z0")
    under the gradin call id, Z_0 of gradW under the gradW call id; Z_1 = U V - Z_0 as usual.
    Returns (gradW triplet, gradin triplet) in core.triplet_gen's (U0, U1, V0, V1, Z0, Z1) order."""
    assert not isinstance(pair, Strong), "mask reuse is not defined for the strong-scaling layout"
    Uf0, Uf1, Vf0, Vf1, _, _ = core.triplet_gen(DEALER_SEED, call_id(pair, step, layer, OP_FWD, 0), B, din, dout, L)
    cgi, cgw = call_id(pair, step, layer, OP_GRADIN, 0), call_id(pair, step, layer, OP_GRADW, 0)
    D0 = core.dealer_prg(L, DEALER_SEED, core.tag("U0"), cgi, B * dout).reshape(B, dout)
    D1 = core.dealer_prg(L, DEALER_SEED, core.tag("U1"), cgi, B * dout).reshape(B, dout)
    Ug = (np.ascontiguousarray(Uf0.T), np.ascontiguousarray(Uf1.T))
    Zg = core.ring_matmul(np.ascontiguousarray((Uf0 + Uf1).T), D0 + D1)
    Zg0 = core.dealer_prg(L, DEALER_SEED, core.tag("Z0"), cgw, din * dout).reshape(din, dout)
    Vi = (np.ascontiguousarray(Vf0.T), np.ascontiguousarray(Vf1.T))
    Zi = core.ring_matmul(D0 + D1, np.ascontiguousarray((Vf0 + Vf1).T))
    Zi0 = core.dealer_prg(L, DEALER_SEED, core.tag("Z0"), cgi, B * din).reshape(B, din)
    return ((Ug[0], Ug[1], D0, D1, Zg0, Zg - Zg0), (D0, D1, Vi[0], Vi[1], Zi0, Zi - Zi0))


def matmul_with(A, B, trip, trunc):
    c = core.beaver_matmul(A, B, trip, trunc=0, l=L)
    return checked_trunc(c, trunc) if trunc else c


def matmul(A, B, pair, step, layer, op, trunc):
    """Beaver product of two shared matrices with the triplet of call id (pair,step,layer,op)."""
    M, K = A[0].shape
    N = B[0].shape[1]
    trip = mat_triplet(pair, step, layer, op, M, K, N)
    c = core.beaver_matmul(A, B, trip, trunc=0, l=L)   # Eq. 6/8, then truncation (R7)
    return checked_trunc(c, trunc) if trunc else c


def relu(z, pair, step, layer, compare="a2b"):
    """Secure ReLU: DReLU by the Kogge-Stone A2B chain (R9) or by the one-round FSS comparison
    (compare="fss", R22: material keyed by the same call id), then one Beaver Hadamard."""
    n = z[0].size
    ht = had_triplet(pair, step, layer, 0, n)
    mat = cmp_material(pair, step, layer, OP_RELU_MSB, n, compare)
    flat = (z[0].reshape(-1), z[1].reshape(-1))
    if compare == "fss":
        (r0, r1), (d0, d1) = core.secure_relu_fss(flat, mat, ht, L)
    else:
        (r0, r1), (d0, d1) = core.secure_relu(flat, mat, ht, L)
    if DIAG["on"]:   # DReLU = 1 - MSB(x) must equal [x >= 0] on the plaintext
        x = _signed(z[0].reshape(-1) + z[1].reshape(-1))
        dr = np.asarray(d0 + d1, dtype=np.uint64)
        DIAG["msb_checked"] += int(x.size)
        DIAG["msb_fail"] += int(np.count_nonzero(dr != (x >= 0).astype(np.uint64)))
    s = z[0].shape
    return (r0.reshape(s), r1.reshape(s)), (d0.reshape(s), d1.reshape(s))


def eq9(z, pair, step, layer, compare="a2b"):
    n = z[0].size
    ht = had_triplet(pair, step, layer, 2, 2 * n, parts=2)
    mat = cmp_material(pair, step, layer, OP_EQ9_MSB, 2 * n, compare, parts=2)
    if compare == "fss":   # Eq. 9 = ReLU(x + 1/2) - ReLU(x - 1/2) with the FSS ReLU (R22)
        x = core.eq9_inputs(z, L, F)
        (r0, r1), _ = core.secure_relu_fss(x, mat, ht, L)
        shape = np.shape(z[0])
        y = (((r0[:n] - r0[n:]) & MASK).reshape(shape), ((r1[:n] - r1[n:]) & MASK).reshape(shape))
    else:
        y = core.secure_eq9(z, mat, ht, L, F)
    if DIAG["on"]:   # Eq. 9 on the grid: clamp(x + 2^(F-1), 0, 2^F) exactly (R8)
        x = _signed(z[0] + z[1])
        want = np.clip(x + (1 << (F - 1)), 0, 1 << F)
        DIAG["msb_checked"] += int(x.size)
        DIAG["msb_fail"] += int(np.count_nonzero(_signed(y[0] + y[1]) != want))
    return y


def hadamard(a, b, pair, step, layer, slot):
    n = a[0].size
    ht = had_triplet(pair, step, layer, slot, n)
    c0, c1 = core.beaver_hadamard((a[0].reshape(-1), a[1].reshape(-1)),
                                  (b[0].reshape(-1), b[1].reshape(-1)), ht, L)
    return c0.reshape(a[0].shape), c1.reshape(a[0].shape)


# --- CNN conv layer as im2col ring GEMM, masked in the un-expanded domain (R17) -------------
def conv_triplet(pair, step, op, B, transpose):
    """U over the raw input (B x C*H*W), V, Z = im2col(U).V (op 0) or im2col(U)^T.V (op 1)."""
    g = CNN_GEOM
    assert not isinstance(pair, Strong), "the strong-scaling layout is not defined for the CNN"
    cid = call_id(pair, step, 0, op, 0)
    nin = B * g["C"] * g["H"] * g["W"]
    rows = B * (g["H"] - g["k"] + 1) * (g["W"] - g["k"] + 1)
    kk = g["C"] * g["k"] * g["k"]
    vshape = (rows, g["Cout"]) if transpose else (kk, g["Cout"])
    U0 = core.dealer_prg(L, DEALER_SEED, core.tag("U0"), cid, nin).reshape(B, -1)
    U1 = core.dealer_prg(L, DEALER_SEED, core.tag("U1"), cid, nin).reshape(B, -1)
    nv = vshape[0] * vshape[1]
    V0 = core.dealer_prg(L, DEALER_SEED, core.tag("V0"), cid, nv).reshape(vshape)
    V1 = core.dealer_prg(L, DEALER_SEED, core.tag("V1"), cid, nv).reshape(vshape)
    Ucol = core.im2col(U0 + U1, g["C"], g["H"], g["W"], g["k"])
    Z = core.ring_matmul(np.ascontiguousarray(Ucol.T) if transpose else Ucol, V0 + V1)
    Z0 = core.dealer_prg(L, DEALER_SEED, core.tag("Z0"), cid, Z.size).reshape(Z.shape)
    return (U0, U1), (V0, V1), (Z0, Z - Z0)


def conv_matmul(X, Bm, U, V, Z, transpose, trunc):
    """C_i = i.E'.F + E'.V_i + U'_i.F + Z_i with E' = im2col(X - U) (^T), U'_i = im2col(U_i) (^T)."""
    g = CNN_GEOM
    col = lambda t: core.im2col(t, g["C"], g["H"], g["W"], g["k"])  # noqa: E731
    tr = (lambda t: np.ascontiguousarray(t.T)) if transpose else (lambda t: t)  # noqa: E731
    E = (X[0] - U[0]) + (X[1] - U[1])                       # Eq. 4 + Eq. 5 on the raw input
    Fm = (Bm[0] - V[0]) + (Bm[1] - V[1])
    Ec = tr(col(E))
    EF = core.ring_matmul(Ec, Fm)
    out = []
    for i in range(2):
        c = i * EF + core.ring_matmul(Ec, V[i]) + core.ring_matmul(tr(col(U[i])), Fm) + Z[i]
        out.append(c)
    return checked_trunc(tuple(out), trunc) if trunc else tuple(out)


# ---------------------------------------------------------------------------------------------
# training step
# ---------------------------------------------------------------------------------------------
def comparison_lt0(t, pair, step, layer, compare="a2b"):
    """Arithmetic shares of [t < 0] (signed) = MSB(t): the A2B chain's MSB (R9), or 1 - DReLU from
    the FSS comparison (R22).  Material keyed like ReLU's (op 3)."""
    n = t[0].size
    mat = cmp_material(pair, step, layer, OP_RELU_MSB, n, compare)
    flat = (t[0].reshape(-1), t[1].reshape(-1))
    if compare == "fss":
        d0, d1 = core.fss_drelu(flat, mat, L)
        out = ((np.uint64(1) - d0) & MASK, (np.uint64(0) - d1) & MASK)
    else:
        out = core.secure_msb(flat, mat, L)
    if DIAG["on"]:
        x = _signed(flat[0] + flat[1])
        DIAG["msb_checked"] += int(x.size)
        DIAG["msb_fail"] += int(np.count_nonzero((out[0] + out[1]) != (x < 0).astype(np.uint64)))
    s = t[0].shape
    return out[0].reshape(s), out[1].reshape(s)


def _svm_forward_backward(model, Xs, Ys, step, pair):
    """Linear SVM, hinge loss, minibatch subgradient (R24; PAPER.md L295 names SVM):
    z = X w;  m = y (.) z;  ind = [m < 1] = [m - 1 < 0];  delta = -(y (.) ind);  gradW = X^T delta."""
    z = matmul(Xs, model.W[0], pair, step, 0, OP_FWD, model.fw[0])
    m = checked_trunc(hadamard(Ys, z, pair, step, 0, 3), F)            # margin, 13 bits
    t = ((m[0] - np.uint64(1 << F)) & MASK, m[1])                       # m - 1 (party 0)
    ind = comparison_lt0(t, pair, step, 0, model.compare)
    c = hadamard(Ys, ind, pair, step, 0, 4)                             # y (.) ind, 13 bits
    delta = ((np.uint64(0) - c[0]) & MASK, (np.uint64(0) - c[1]) & MASK)
    grads = [matmul(_T(Xs), delta, pair, step, 0, OP_GRADW, 0)]
    return grads, z


def _rnn_forward(model, Xs, step, pair):
    """Elman RNN (R25; "passes the states in its own network"):
    h_0 = 0;  A_t = [x_t | h_{t-1}];  z_t = trunc(A_t . W_1, f_w);  h_t = ReLU(z_t)  (t = 1..T,
    call-id layer t);  yhat = Eq9(trunc(h_T . W_o, f_w))  (layer T + 1)."""
    g = RNN_GEOM
    T, D, H = g["T"], g["D"], g["H"]
    B = Xs[0].shape[0]
    h = (np.zeros((B, H), np.uint64), np.zeros((B, H), np.uint64))
    As, drelus = [], []
    for t in range(1, T + 1):
        A = tuple(np.ascontiguousarray(np.concatenate([x[:, (t - 1) * D:t * D], hh], axis=1)) for x, hh in zip(Xs, h))
        z = matmul(A, model.W[0], pair, step, t, OP_FWD, model.fw[0])
        h, d = relu(z, pair, step, t, model.compare)
        As.append(A)
        drelus.append(d)
    zo = matmul(h, model.W[1], pair, step, T + 1, OP_FWD, model.fw[1])
    return As, drelus, h, zo


def _rnn_forward_backward(model, Xs, Ys, step, pair):
    """Backpropagation through time: gW_o = h_T^T delta; delta_T = trunc(delta . W_o^T) (.) DReLU_T;
    gW_1 = sum_t A_t^T delta_t (untruncated, ring addition); delta_{t-1} = trunc(delta_t . W_h^T)
    (.) DReLU_{t-1} with W_h = the last H rows of W_1."""
    g = RNN_GEOM
    T, D = g["T"], g["D"]
    As, drelus, h, zo = _rnn_forward(model, Xs, step, pair)
    yhat = eq9(zo, pair, step, T + 1, model.compare)
    delta = sub_pair(yhat, Ys)
    gWo = matmul(_T(h), delta, pair, step, T + 1, OP_GRADW, 0)
    t_ = matmul(delta, _T(model.W[1]), pair, step, T + 1, OP_GRADIN, model.fw[1])
    delta = hadamard(t_, drelus[T - 1], pair, step, T, 1)
    gW1 = (np.zeros(model.W[0][0].shape, np.uint64), np.zeros(model.W[0][0].shape, np.uint64))
    for t in range(T, 0, -1):
        gt = matmul(_T(As[t - 1]), delta, pair, step, t, OP_GRADW, 0)
        gW1 = (gW1[0] + gt[0], gW1[1] + gt[1])
        if t > 1:
            Wh = tuple(np.ascontiguousarray(w[D:, :]) for w in model.W[0])
            t_ = matmul(delta, _T(Wh), pair, step, t, OP_GRADIN, model.fw[0])
            delta = hadamard(t_, drelus[t - 2], pair, step, t - 1, 1)
    return [gW1, gWo], yhat


def forward_backward(model, Xs, Ys, step, pair=0):
    """Returns (per-layer untruncated weight-gradient shares, prediction shares)."""
    task = model.task
    if task == "cnn":
        return _cnn_forward_backward(model, Xs, Ys, step, pair)
    if task == "svm":
        return _svm_forward_backward(model, Xs, Ys, step, pair)
    if task == "rnn":
        return _rnn_forward_backward(model, Xs, Ys, step, pair)
    nl = len(model.W)
    acts = [Xs]
    drelus = []
    h = Xs
    for layer in range(nl):
        z = matmul(h, model.W[layer], pair, step, layer, OP_FWD, model.fw[layer])
        if layer < nl - 1:
            h, d = relu(z, pair, step, layer, model.compare)
            drelus.append(d)
            acts.append(h)
        elif task == "linreg":
            h = z
        else:
            h = eq9(z, pair, step, layer, model.compare)
    yhat = h
    delta = sub_pair(yhat, Ys)
    grads = [None] * nl
    B = Xs[0].shape[0]
    for layer in range(nl - 1, -1, -1):
        if model.mask_reuse:
            din, dout = model.W[layer][0].shape
            tg, ti = reuse_triplets(pair, step, layer, B, din, dout)
            grads[layer] = matmul_with(_T(acts[layer]), delta, tg, 0)
            if layer > 0:
                t = matmul_with(delta, _T(model.W[layer]), ti, model.fw[layer])
                delta = hadamard(t, drelus[layer - 1], pair, step, layer - 1, 1)
            continue
        grads[layer] = matmul(_T(acts[layer]), delta, pair, step, layer, OP_GRADW, 0)
        if layer > 0:
            t = matmul(delta, _T(model.W[layer]), pair, step, layer, OP_GRADIN, model.fw[layer])
            delta = hadamard(t, drelus[layer - 1], pair, step, layer - 1, 1)
    return grads, yhat


def _cnn_forward_backward(model, Xs, Ys, step, pair):
    g = CNN_GEOM
    B = Xs[0].shape[0]
    U, V, Z = conv_triplet(pair, step, OP_FWD, B, transpose=False)
    # forward conv: V for op 0 is the weight mask (75 x 16), Z = im2col(U) . V
    fw = model.fw
    zc = conv_matmul(Xs, model.W[0], U, V, Z, transpose=False, trunc=fw[0])   # (B*784) x 16
    h1, d1 = relu(zc, pair, step, 0, model.compare)
    h1 = (h1[0].reshape(B, -1), h1[1].reshape(B, -1))                         # B x 12544
    z2 = matmul(h1, model.W[1], pair, step, 1, OP_FWD, fw[1])
    h2, d2 = relu(z2, pair, step, 1, model.compare)
    z3 = matmul(h2, model.W[2], pair, step, 2, OP_FWD, fw[2])
    yhat = eq9(z3, pair, step, 2, model.compare)
    delta = sub_pair(yhat, Ys)
    grads = [None] * 3
    grads[2] = matmul(_T(h2), delta, pair, step, 2, OP_GRADW, 0)
    t = matmul(delta, _T(model.W[2]), pair, step, 2, OP_GRADIN, fw[2])
    delta = hadamard(t, d2, pair, step, 1, 1)
    grads[1] = matmul(_T(h1), delta, pair, step, 1, OP_GRADW, 0)
    t = matmul(delta, _T(model.W[1]), pair, step, 1, OP_GRADIN, fw[1])
    d1f = (d1[0].reshape(B, -1), d1[1].reshape(B, -1))
    delta = hadamard(t, d1f, pair, step, 0, 1)
    rows = B * (g["H"] - g["k"] + 1) * (g["W"] - g["k"] + 1)
    delta = (delta[0].reshape(rows, g["Cout"]), delta[1].reshape(rows, g["Cout"]))
    U, V, Z = conv_triplet(pair, step, OP_GRADW, B, transpose=True)
    grads[0] = conv_matmul(Xs, delta, U, V, Z, transpose=True, trunc=0)
    return grads, yhat


def apply_update(model, grads, n_pairs=1):
    """W^m_i -= trunc_i(gradW_i, 2F + LR_SHIFT - MASTER + log2(n_pairs)); W_i = trunc_i(W^m_i,
    MASTER - f_w)  (R14, R21)."""
    extra = int(np.log2(n_pairs))
    assert (1 << extra) == n_pairs
    for layer, g in enumerate(grads):
        gt = checked_trunc(g, 2 * F + LR_SHIFT - MASTER + extra)
        if model.task == "svm":   # weight decay: W^m -= trunc(W^m, WD_SHIFT) (R24), from the old W^m
            gt = (gt[0] + trunc_pair(model.Wm[layer], WD_SHIFT)[0], gt[1] + trunc_pair(model.Wm[layer], WD_SHIFT)[1])
        model.Wm[layer] = sub_pair(model.Wm[layer], gt)
        model.W[layer] = checked_trunc(model.Wm[layer], MASTER - model.fw[layer])


def strong_forward_backward(model, Xs, Ys, step, P):
    """Strong scaling over P pairs (R28), every pair simulated: Xs / Ys are
    the global batch's shares; pair k runs forward / backward on rows [k b, (k + 1) b) with the
    Strong(k, P) material, and each party's weight-gradient shares are summed over the P pairs
    (the per-party all-reduce; ring addition, exact).  The sum is the global batch's gradient, so
    the update takes no extra shift (apply_update(..., n_pairs=1)).  Returns (summed gradient
    shares, per-pair prediction shares stacked in row order)."""
    B = Xs[0].shape[0]
    assert B % P == 0
    b = B // P
    total, yh = None, []
    for k in range(P):
        r = slice(k * b, (k + 1) * b)
        g, y = forward_backward(model, (Xs[0][r], Xs[1][r]), (Ys[0][r], Ys[1][r]), step, Strong(k, P))
        total = g if total is None else [(t[0] + u[0], t[1] + u[1]) for t, u in zip(total, g)]
        yh.append(y)
    return total, (np.concatenate([y[0] for y in yh]), np.concatenate([y[1] for y in yh]))


def train_step(model, X, Y, step, pair=0):
    Xs, Ys = share_batch(X, Y, step, pair)
    grads, yhat = forward_backward(model, Xs, Ys, step, pair)
    apply_update(model, grads)
    return yhat


def infer(model, Xs, step, pair=0):
    """Secure inference = the forward half."""
    task = model.task
    if task == "rnn":
        _, _, _, zo = _rnn_forward(model, Xs, step, pair)
        return eq9(zo, pair, step, RNN_GEOM["T"] + 1, model.compare)
    if task == "cnn":
        B = Xs[0].shape[0]
        U, V, Z = conv_triplet(pair, step, OP_FWD, B, transpose=False)
        zc = conv_matmul(Xs, model.W[0], U, V, Z, transpose=False, trunc=model.fw[0])
        h, _ = relu(zc, pair, step, 0, model.compare)
        h = (h[0].reshape(B, -1), h[1].reshape(B, -1))
        for layer in (1, 2):
            z = matmul(h, model.W[layer], pair, step, layer, OP_FWD, model.fw[layer])
            h = relu(z, pair, step, layer, model.compare)[0] if layer == 1 else eq9(z, pair, step, layer, model.compare)
        return h
    h = Xs
    nl = len(model.W)
    for layer in range(nl):
        z = matmul(h, model.W[layer], pair, step, layer, OP_FWD, model.fw[layer])
        if layer < nl - 1:
            h = relu(z, pair, step, layer, model.compare)[0]
        elif task in ("linreg", "svm"):   # SVM inference: w^T x
            h = z
        else:
            h = eq9(z, pair, step, layer, model.compare)
    return h
