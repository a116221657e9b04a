"""GPU parity of the one-round FSS comparison (R22) against the oracle,
through the C ABI (gpu).  Bar: bit-exact for every dealer word, opened value and share."""
import numpy as np
import pytest
import torch

from tests.util import to_np

pytestmark = pytest.mark.gpu
SEED = 0x50534D4C


@pytest.fixture(scope="module")
def P():
    from paper_conf_icpp_chenzzzz020_b200 import build, psml
    build.build()
    return psml


@pytest.fixture(scope="module")
def ctx(P):
    c = P.Ctx(l=64, frac_bits=13, backend=1)
    yield c
    c.close()


def _x(orc, n, salt):
    x = orc.prg(64, SEED, orc.tag("fx"), salt, n) >> np.uint64(20)
    x = np.where(np.arange(n) % 3 == 0, np.uint64(0) - x, x).astype(np.uint64)
    edges = np.array([0, 1, (1 << 63) - 1, 1 << 63, (1 << 64) - 1, 1 << 12, (1 << 64) - (1 << 12)], dtype=np.uint64)
    x[:min(n, edges.size)] = edges[:min(n, edges.size)]
    x0 = orc.prg(64, SEED + 1, orc.tag("xs"), salt, n)
    return x, (x0, x - x0)


def _dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


@pytest.mark.parametrize("n", [1, 7, 129, 4099, 65537])
def test_fss_dealer_bitexact(P, orc, n):
    mat = P.fss_dealer(P.Ring(64, 13), SEED + 2, 0x0102030405060708, n)
    torch.cuda.synchronize()
    want = orc.fss_dealer(SEED + 2, 0x0102030405060708, n)
    for p in range(2):
        assert np.array_equal(to_np(mat[p]), want[p]), p


@pytest.mark.parametrize("n", [1, 33, 4099, 65537])
def test_fss_drelu_bitexact(P, orc, ctx, n):
    x, xs = _x(orc, n, n)
    mat = orc.fss_dealer(SEED + 3, 9, n)
    d, xh = P.secure_drelu_fss(ctx, (_dev(xs[0]), _dev(xs[1])), (_dev(mat[0]), _dev(mat[1])), trace=True)
    torch.cuda.synchronize()
    (w0, w1), wxh = orc.fss_drelu(xs, mat, trace=True)
    assert np.array_equal(to_np(xh), wxh)
    assert np.array_equal(to_np(d[0]), w0) and np.array_equal(to_np(d[1]), w1)
    signed = x.view(np.int64)
    assert np.array_equal(w0 + w1, (signed >= 0).astype(np.uint64))


@pytest.mark.parametrize("n", [5, 16384])
def test_fss_relu_bitexact_and_split_form(P, orc, ctx, n):
    x, xs = _x(orc, n, 1000 + n)
    mat = orc.fss_dealer(SEED + 4, 10, n)
    ht = orc.hadamard_triplet_gen(SEED + 5, 11, n)
    dv = [_dev(t) for t in ht]
    y, d = P.secure_relu_fss(ctx, (_dev(xs[0]), _dev(xs[1])), (_dev(mat[0]), _dev(mat[1])), dv[0:2], dv[2:4], dv[4:6])
    torch.cuda.synchronize()
    (r0, r1), (d0, d1) = orc.secure_relu_fss(xs, mat, ht)
    assert np.array_equal(to_np(y[0]), r0) and np.array_equal(to_np(y[1]), r1)
    assert np.array_equal(to_np(d[0]), d0) and np.array_equal(to_np(d[1]), d1)
    # split deployment form: each party masks alone, the messages are exchanged, each opens alone
    msgs = [P.fss_mask(ctx, p, _dev(xs[p]), _dev(mat[p])) for p in range(2)]
    dd = [P.fss_open_drelu(ctx, p, msgs[p], msgs[1 - p], _dev(mat[p])) for p in range(2)]
    torch.cuda.synchronize()
    assert np.array_equal(to_np(dd[0]), d0) and np.array_equal(to_np(dd[1]), d1)


# --- the FSS comparison inside training (psml_model_desc.compare = 1) ------------------------------
def _compare_shares(tr, om):
    for layer in range(len(om.Wm)):
        g0, g1 = tr.master_shares(layer)
        assert np.array_equal(to_np(g0).reshape(om.Wm[layer][0].shape), om.Wm[layer][0]), layer
        assert np.array_equal(to_np(g1).reshape(om.Wm[layer][1].shape), om.Wm[layer][1]), layer


@pytest.mark.parametrize("task,steps", [("logreg", 2), ("svm", 2), ("mlp", 2), ("rnn", 1)])
def test_training_with_fss_comparison_bitexact(P, task, steps):
    """Every ReLU / Eq. 9 of the step through the one-round FSS comparison: eager steps and
    CUDA-graph replays (dealer inside the graph) bit-exact vs the oracle's protocol."""
    import synth
    from oracle import protocol as OP
    from paper_conf_icpp_chenzzzz020_b200.train import SecureTrainer
    Wi = synth.init_weights(task)
    tr = SecureTrainer(task, Wi, backend=1, compare="fss")
    om = OP.Model(task, Wi, compare="fss")
    X, Y = synth.batch(task, 0)
    tr.step(torch.from_numpy(X), torch.from_numpy(Y), 0)
    OP.train_step(om, X, Y, 0)
    torch.cuda.synchronize()
    _compare_shares(tr, om)
    if steps > 1:
        tr.capture(pipelined=True)
        for s in range(1, steps + 1):
            X, Y = synth.batch(task, s)
            tr.graph_step(torch.from_numpy(X), torch.from_numpy(Y), s)
            OP.train_step(om, X, Y, s)
            torch.cuda.synchronize()
            _compare_shares(tr, om)
    tr.close()
