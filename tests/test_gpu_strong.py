"""Strong scaling on the GPU (R28) vs the oracle, bit-exact.

P co-resident pairs on the one GPU stand for P GPUs: pair k trains rows [k b, (k + 1) b) of the
global batch with the row-sliced dealer layout (psml_model_desc.strong_pairs = P); the per-party
all-reduce of the untruncated gradient shares over the pairs is a ring sum of their gradient
buffers (what NCCL's ncclSum on uint64 does across GPUs); every pair updates with extra_shift 0.
After every step each pair's prediction shares equal the oracle's rows and every pair's master
shares equal the oracle's (oracle/protocol.strong_forward_backward).
"""
import numpy as np
import pytest
import torch

import synth
from oracle import protocol as OP
from tests.util import to_dev, to_np

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def T():
    from paper_conf_icpp_chenzzzz020_b200 import build, train
    build.build()
    return train


def _compare_master(tr, om):
    for layer in range(len(om.Wm)):
        g0, g1 = tr.master_shares(layer)
        assert np.array_equal(to_np(g0).reshape(om.Wm[layer][0].shape), om.Wm[layer][0]), layer
        assert np.array_equal(to_np(g1).reshape(om.Wm[layer][1].shape), om.Wm[layer][1]), layer


def _strong_step(trs, Xs, Ys, step, b):
    for k, tr in enumerate(trs):
        r = slice(k * b, (k + 1) * b)
        tr.model.deal(step)
        tr.model.forward_backward((to_dev(Xs[0][r]), to_dev(Xs[1][r])), (to_dev(Ys[0][r]), to_dev(Ys[1][r])), step)
    total = trs[0].grad_tensor().clone()
    for tr in trs[1:]:
        total += tr.grad_tensor()            # int64 two's-complement sum == Z_2^64 addition
    for tr in trs:
        tr.grad_tensor().copy_(total)
        tr.model.apply_update(extra_shift=tr.update_shift(len(trs)))


@pytest.mark.parametrize("task,compare,pairs,steps", [("linreg", "a2b", 4, 2), ("logreg", "a2b", 4, 2),
                                                      ("mlp", "a2b", 4, 3), ("mlp", "fss", 2, 2),
                                                      ("svm", "a2b", 4, 2), ("rnn", "a2b", 2, 2),
                                                      ("mlp", "a2b", 16, 1)])
def test_strong_scaling_bitexact_vs_oracle(T, task, compare, pairs, steps):
    Wi = synth.init_weights(task)
    b = 128 // pairs
    trs = [T.SecureTrainer(task, Wi, batch=b, pair_id=k, strong_pairs=pairs, compare=compare) for k in range(pairs)]
    om = OP.Model(task, Wi, compare=compare)
    for s in range(steps):
        X, Y = synth.batch(task, s)
        Xs, Ys = OP.share_batch(X, Y, s)
        grads, yo = OP.strong_forward_backward(om, Xs, Ys, s, pairs)
        OP.apply_update(om, grads, n_pairs=1)
        _strong_step(trs, Xs, Ys, s, b)
        torch.cuda.synchronize()
        for k, tr in enumerate(trs):
            y0, y1 = tr.last_yhat()
            r = slice(k * b, (k + 1) * b)
            assert np.array_equal(to_np(y0).reshape(yo[0][r].shape), yo[0][r]), (s, k)
            assert np.array_equal(to_np(y1).reshape(yo[1][r].shape), yo[1][r]), (s, k)
            _compare_master(tr, om)
    for tr in trs:
        tr.close()


def test_strong_step1_rows_of_single_pair_run(T):
    """SURVEY 8(c) multi-GPU pin (2) on the GPU: step 1 of the 4-pair run has prediction shares
    that are bit-identical row-slices of the 1-pair run, and its all-reduced untruncated gradient
    reconstructs to the 1-pair gradient exactly."""
    task, pairs = "mlp", 4
    Wi = synth.init_weights(task)
    X, Y = synth.batch(task, 0)
    Xs, Ys = OP.share_batch(X, Y, 0)
    one = T.SecureTrainer(task, Wi)
    one.model.deal(0)
    one.model.forward_backward((to_dev(Xs[0]), to_dev(Xs[1])), (to_dev(Ys[0]), to_dev(Ys[1])), 0)
    b = 128 // pairs
    trs = [T.SecureTrainer(task, Wi, batch=b, pair_id=k, strong_pairs=pairs) for k in range(pairs)]
    for k, tr in enumerate(trs):
        r = slice(k * b, (k + 1) * b)
        tr.model.deal(0)
        tr.model.forward_backward((to_dev(Xs[0][r]), to_dev(Xs[1][r])), (to_dev(Ys[0][r]), to_dev(Ys[1][r])), 0)
    torch.cuda.synchronize()
    y1 = [to_np(t) for t in one.last_yhat()]
    ys = [np.concatenate([to_np(tr.last_yhat()[p]) for tr in trs]) for p in (0, 1)]
    assert np.array_equal(ys[0], y1[0]) and np.array_equal(ys[1], y1[1])
    g1 = to_np(one.grad_tensor()).reshape(2, -1)
    gs = sum(tr.grad_tensor().clone() for tr in trs).cpu().numpy().astype(np.uint64).reshape(2, -1)
    assert np.array_equal(g1[0] + g1[1], gs[0] + gs[1])
    assert not np.array_equal(g1[0], gs[0])   # per-pair weight-gradient triplets: other shares
    for tr in trs + [one]:
        tr.close()


def test_strong_scaling_rejects_bad_layouts(T):
    from paper_conf_icpp_chenzzzz020_b200 import psml
    Wi = synth.init_weights("mlp")
    with pytest.raises(psml.PsmlError):
        T.SecureTrainer("mlp", Wi, batch=12, pair_id=0, strong_pairs=4)      # rows not a multiple of 8
    with pytest.raises(psml.PsmlError):
        T.SecureTrainer("mlp", Wi, batch=32, pair_id=4, strong_pairs=4)      # pair outside the group
    with pytest.raises(psml.PsmlError):
        T.SecureTrainer("mlp", Wi, batch=32, pair_id=0, strong_pairs=4, mask_reuse=True)
    with pytest.raises(psml.PsmlError):
        T.SecureTrainer("cnn", synth.init_weights("cnn"), batch=32, pair_id=0, strong_pairs=4)
    tr = T.SecureTrainer("mlp", Wi, batch=32, pair_id=0, strong_pairs=4)
    with pytest.raises(ValueError):
        tr.update_shift(2)
    assert tr.update_shift(4) == 0
    tr.close()
