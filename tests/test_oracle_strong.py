"""Pins of the oracle's strong-scaling layout (R28; not gpu).

P pairs train on ONE global batch, pair k on rows [k b, (k + 1) b).  What the mathematics fixes:
  * the forward pass is row-wise, so with the row-slice dealer layout every pair's prediction
    shares are exactly the rows of the single-pair run's shares (same material, same openings);
  * the per-party sum of the pairs' weight-gradient shares reconstructs to sum_k A_k^T delta_k =
    A^T delta, i.e. EXACTLY the single-pair gradient (ring addition), although the shares differ
    (the weight-gradient triplets are independent per pair);
  * training with the summed gradient and no extra shift tracks fp64 SGD on the global batch.
"""
import numpy as np
import pytest

import synth
from oracle import core, plain
from oracle import protocol as P


def _same(a, b):
    return all(np.array_equal(np.asarray(x).reshape(-1), np.asarray(y).reshape(-1)) for x, y in zip(a, b))


@pytest.mark.parametrize("task,compare,pairs", [("linreg", "a2b", 4), ("logreg", "a2b", 4), ("mlp", "a2b", 4),
                                                ("mlp", "fss", 2), ("svm", "a2b", 4), ("rnn", "a2b", 2)])
def test_strong_step_identities(task, compare, pairs):
    Wi = synth.init_weights(task)
    X, Y = synth.batch(task, 0)
    Xs, Ys = P.share_batch(X, Y, 5)
    one = P.Model(task, Wi, compare=compare)
    g1, y1 = P.forward_backward(one, Xs, Ys, 5, 0)
    many = P.Model(task, Wi, compare=compare)
    gs, ys = P.strong_forward_backward(many, Xs, Ys, 5, pairs)
    assert _same(ys, y1), "forward shares are not the row-slices of the single-pair run"
    for layer, (a, b) in enumerate(zip(gs, g1)):
        assert np.array_equal(core.reconstruct(*a), core.reconstruct(*b)), layer
    # the weight-gradient triplets are per pair: the summed shares differ from the 1-pair shares
    assert not np.array_equal(gs[0][0], g1[0][0])


def test_strong_slices_are_disjoint_and_cover():
    """Every global element is owned by exactly one pair, per part (Eq. 9's two halves)."""
    n, Pn = 24, 4
    for parts in (1, 2):
        idx = np.concatenate([P._slice_idx(P.Strong(k, Pn), n, parts) for k in range(Pn)])
        assert sorted(idx.tolist()) == list(range(Pn * n))
    # pair 1 of 2, Eq. 9 layout [z + 1/2 ; z - 1/2] of 3 rows each: rows 3..5 of both halves
    assert P._slice_idx(P.Strong(1, 2), 6, 2).tolist() == [3, 4, 5, 9, 10, 11]


@pytest.mark.parametrize("task,steps,pairs,tol_log2", [("logreg", 30, 4, -16), ("mlp", 6, 4, -15)])
def test_strong_training_tracks_fp64(task, steps, pairs, tol_log2):
    Wi = synth.init_weights(task)
    m, pm = P.Model(task, Wi), plain.PlainModel(task, Wi)
    for s in range(steps):
        X, Y = synth.batch(task, s)
        Xs, Ys = P.share_batch(X, Y, s)
        grads, _ = P.strong_forward_backward(m, Xs, Ys, s, pairs)
        P.apply_update(m, grads, n_pairs=1)
        pm.step(X, Y)
    err = max(np.abs(a - b).max() for a, b in zip(m.decoded_master(), pm.W))
    assert err < 2.0 ** tol_log2, np.log2(err)


def test_strong_layout_rejects_cnn_and_mask_reuse():
    with pytest.raises(AssertionError):
        P.conv_triplet(P.Strong(0, 2), 0, P.OP_FWD, 8, False)
    with pytest.raises(AssertionError):
        P.reuse_triplets(P.Strong(0, 2), 0, 0, 8, 4, 4)
