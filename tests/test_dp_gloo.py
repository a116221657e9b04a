"""Data-parallel host logic on CPU with world_size-2 gloo (not gpu).

Two processes, one party pair each, run the oracle's forward/backward on their own rows (pair id
in the call ids, R16), sum their untruncated gradient shares with the product's
`parallel.ring_allreduce_` (int64 two's-complement SUM == Z_2^64 addition) and apply the update
with log2(2) extra truncation bits.  Both ranks must end bit-identical to a single-process
reference that sums the two pairs' gradients in numpy uint64.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _flatten(grads):
    return np.concatenate([np.concatenate([g[i].reshape(-1) for g in grads]) for i in (0, 1)])


def _unflatten(flat, like):
    out, off = [], 0
    P = sum(g[0].size for g in like)
    for g in like:
        n = g[0].size
        out.append((flat[off:off + n].reshape(g[0].shape).copy(),
                    flat[P + off:P + off + n].reshape(g[0].shape).copy()))
        off += n
    return out


def _worker(rank, world, port, task, outdir):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import synth
    from oracle import protocol as OP
    from paper_conf_icpp_chenzzzz020_b200.parallel import dp_update_shift, ring_allreduce_
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    m = OP.Model(task, synth.init_weights(task))
    for step in range(2):
        X, Y = synth.batch(task, step, pair=rank, n_pairs=world)
        Xs, Ys = OP.share_batch(X, Y, step, pair=rank)
        grads, _ = OP.forward_backward(m, Xs, Ys, step, pair=rank)
        flat = torch.from_numpy(_flatten(grads))
        ring_allreduce_(flat)
        OP.apply_update(m, _unflatten(flat.numpy(), grads), n_pairs=1 << dp_update_shift(world))
    np.savez(os.path.join(outdir, f"rank{rank}.npz"),
             *[w for pair in m.Wm for w in pair])
    # wrap-around check of the all-reduce itself
    big = torch.tensor([2 ** 63 - 1 - rank, 2 ** 64 - 1, 5], dtype=torch.uint64)
    ring_allreduce_(big)
    np.save(os.path.join(outdir, f"big{rank}.npy"), big.numpy())
    dist.destroy_process_group()


@pytest.mark.parametrize("task", ["linreg", "mlp"])
def test_dp_two_pairs_gloo_matches_single_process_sum(tmp_path, task):
    import synth
    from oracle import protocol as OP
    world = 2
    mp.spawn(_worker, args=(world, _free_port(), task, str(tmp_path)), nprocs=world, join=True)
    # single-process reference: both pairs' gradients summed in numpy uint64
    m = OP.Model(task, synth.init_weights(task))
    for step in range(2):
        total = None
        for pair in range(world):
            X, Y = synth.batch(task, step, pair=pair, n_pairs=world)
            Xs, Ys = OP.share_batch(X, Y, step, pair=pair)
            grads, _ = OP.forward_backward(m, Xs, Ys, step, pair=pair)
            f = _flatten(grads)
            total = f if total is None else total + f
        OP.apply_update(m, _unflatten(total, grads), n_pairs=world)
    want = [w for pair in m.Wm for w in pair]
    for r in range(world):
        got = np.load(tmp_path / f"rank{r}.npz")
        for i, w in enumerate(want):
            assert np.array_equal(got[f"arr_{i}"], w), (r, i)
        big = np.load(tmp_path / f"big{r}.npy")
        assert big.tolist() == [(2 ** 63 - 1) * 2 - 1, 2 ** 64 - 2, 10]


def _strong_worker(rank, world, port, task, outdir):
    """Pair `rank` of a strong-scaling group (R28): rows [rank b, (rank + 1) b)
    of the global batch, row-sliced material, gradient all-reduce over gloo, no extra shift."""
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import synth
    from oracle import protocol as OP
    from paper_conf_icpp_chenzzzz020_b200.parallel import ring_allreduce_, strong_rows
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    m = OP.Model(task, synth.init_weights(task))
    for step in range(2):
        X, Y = synth.batch(task, step)
        Xs, Ys = OP.share_batch(X, Y, step)          # the client shares the global batch
        r = strong_rows(rank, world, X.shape[0])     # ... and this pair receives its rows
        grads, _ = OP.forward_backward(m, (Xs[0][r], Xs[1][r]), (Ys[0][r], Ys[1][r]), step, OP.Strong(rank, world))
        flat = torch.from_numpy(_flatten(grads))
        ring_allreduce_(flat)
        OP.apply_update(m, _unflatten(flat.numpy(), grads), n_pairs=1)
    np.savez(os.path.join(outdir, f"strong{rank}.npz"), *[w for pair in m.Wm for w in pair])
    dist.destroy_process_group()


def test_strong_dp_two_pairs_gloo_matches_oracle():
    import tempfile

    import synth
    from oracle import protocol as OP
    world, task = 2, "mlp"
    with tempfile.TemporaryDirectory() as d:
        mp.spawn(_strong_worker, args=(world, _free_port(), task, d), nprocs=world, join=True)
        m = OP.Model(task, synth.init_weights(task))
        for step in range(2):
            X, Y = synth.batch(task, step)
            Xs, Ys = OP.share_batch(X, Y, step)
            grads, _ = OP.strong_forward_backward(m, Xs, Ys, step, world)
            OP.apply_update(m, grads, n_pairs=1)
        want = [w for pair in m.Wm for w in pair]
        for r in range(world):
            got = np.load(os.path.join(d, f"strong{r}.npz"))
            for i, w in enumerate(want):
                assert np.array_equal(got[f"arr_{i}"], w), (r, i)


def test_strong_rows():
    from paper_conf_icpp_chenzzzz020_b200.parallel import strong_rows
    assert [strong_rows(k, 4, 128) for k in range(4)] == [slice(0, 32), slice(32, 64), slice(64, 96), slice(96, 128)]
    with pytest.raises(ValueError):
        strong_rows(0, 3, 128)        # 128 rows do not split into 3 pairs
    with pytest.raises(ValueError):
        strong_rows(0, 32, 128)       # 4 rows per pair: not a multiple of 8 (ChaCha20 block slices)


def test_dp_update_shift_and_rows():
    from paper_conf_icpp_chenzzzz020_b200.parallel import dp_update_shift, pair_rows
    import synth
    assert [dp_update_shift(w) for w in (1, 2, 4, 8)] == [0, 1, 2, 3]
    with pytest.raises(ValueError):
        dp_update_shift(3)
    # the product's row sharding matches the synthetic-data generator's
    for step, pair in [(0, 0), (3, 1), (467, 3)]:
        start = pair_rows(step, pair, 4, 128, 60000)
        X, _ = synth.batch("mlp", step, 128, pair=pair, n_pairs=4)
        assert np.array_equal(X, synth.rows("mnist", start, 128))


def test_split_pair_layout():
    """Split deployment placement: pair k = (rank k: party 0, rank k + N/2: party 1);
    each rank's peer is the other party of its pair; odd world sizes are rejected."""
    from paper_conf_icpp_chenzzzz020_b200.parallel import pair_layout
    of = pair_layout(8)
    assert [of(r) for r in range(8)] == [(0, 0, 4), (0, 1, 5), (0, 2, 6), (0, 3, 7),
                                         (1, 0, 0), (1, 1, 1), (1, 2, 2), (1, 3, 3)]
    assert pair_layout(2)(1) == (1, 0, 0)
    for bad in (1, 3):
        with pytest.raises(ValueError):
            pair_layout(bad)
