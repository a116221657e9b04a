"""Pins of the oracle's one-round FSS comparison (R22), not gpu.

The DCF (Boyle et al., EUROCRYPT 2021, Fig. 1) is pinned by its defining property, checked by
brute force over every input of small domains: Eval(0, k_0, x) + Eval(1, k_1, x) = beta * [x < alpha]
in Z_{2^l}.  The DReLU built on it is pinned exhaustively on toy rings against the sign bit of the
reconstructed input, and on l = 64 edge values."""
import numpy as np
import pytest


def _mask(l):
    return (1 << l) - 1


@pytest.mark.parametrize("l,n_bits", [(8, 7), (16, 8), (64, 8), (32, 10)])
def test_dcf_exhaustive(orc, l, n_bits):
    rng = np.random.default_rng(l * 100 + n_bits)
    for trial in range(6):
        alpha = int(rng.integers(0, 1 << n_bits)) if trial else 0
        if trial == 1:
            alpha = (1 << n_bits) - 1
        beta = int(rng.integers(0, 1 << min(l, 63))) & _mask(l)
        s0 = tuple(int(v) for v in rng.integers(0, 1 << 63, 2, dtype=np.uint64))
        s1 = tuple(int(v) for v in rng.integers(0, 1 << 63, 2, dtype=np.uint64))
        k0, k1 = orc.dcf_gen(l, n_bits, alpha, beta, s0, s1)
        assert np.array_equal(k0[2:], k1[2:])          # correction words are common
        for x in range(1 << n_bits):
            y = (orc.dcf_eval(l, n_bits, 0, k0, x) + orc.dcf_eval(l, n_bits, 1, k1, x)) & _mask(l)
            assert y == (beta if x < alpha else 0), (alpha, beta, x)


def test_dcf_single_key_looks_random(orc):
    """A party's own output share alone is not the function value (the shares mask it)."""
    k0, k1 = orc.dcf_gen(16, 8, 100, 1, (1, 2), (3, 4))
    outs = {orc.dcf_eval(16, 8, 0, k0, x) for x in range(256)}
    assert len(outs) > 200


def _signed(v, l):
    v = np.asarray(v, dtype=np.uint64).astype(object) if l == 64 else np.asarray(v, dtype=np.int64)
    return np.where(v >= (1 << (l - 1)), v - (1 << l), v)


@pytest.mark.parametrize("l", [8, 16])
def test_fss_drelu_exhaustive_toy_rings(orc, l):
    """Every x of Z_{2^l}, 3 dealer seeds x random share splits: DReLU shares reconstruct to
    [x >= 0] (signed), and the only opened value is xhat = x + r."""
    n = 1 << l
    x = np.arange(n, dtype=np.uint64)
    for seed in (5, 6, 7):
        x0 = orc.prg(l, seed, orc.tag("xs"), 1, n)
        x1 = (x - x0) & np.uint64(_mask(l))
        mat = orc.fss_dealer(seed, 77, n, l)
        (d0, d1), xh = orc.fss_drelu((x0, x1), mat, l, trace=True)
        d = (d0 + d1) & np.uint64(_mask(l))
        want = (_signed(x, l) >= 0).astype(np.uint64)
        assert np.array_equal(d, want)
        r = (mat[0][:n] + mat[1][:n]) & np.uint64(_mask(l))
        assert np.array_equal(xh, (x + r) & np.uint64(_mask(l)))


def test_fss_drelu_l64_edges_and_random(orc):
    l = 64
    edges = [0, 1, 2, (1 << 63) - 1, 1 << 63, (1 << 63) + 1, (1 << 64) - 1, 1 << 12, (1 << 64) - (1 << 12),
             1 << 13, (1 << 64) - (1 << 13)]
    rnd = [int(v) for v in orc.prg(64, 9, orc.tag("rx"), 0, 2000)]
    x = np.array(edges + rnd, dtype=np.uint64)
    x0 = orc.prg(64, 3, orc.tag("xs"), 2, x.size)
    x1 = x - x0
    mat = orc.fss_dealer(0x50534D4E, 5, x.size)
    d0, d1 = orc.fss_drelu((x0, x1), mat)
    got = d0 + d1
    want = np.array([1 if v < (1 << 63) else 0 for v in x.tolist()], dtype=np.uint64)
    assert np.array_equal(got, want)


def test_secure_relu_fss_matches_a2b_relu(orc):
    """ReLU through the FSS comparison reconstructs to the same values as the A2B-chain ReLU
    (both exact on the grid), for l = 64."""
    n = 4096
    x = orc.prg(64, 11, orc.tag("rl"), 0, n) >> np.uint64(40)
    x = np.where(np.arange(n) % 2 == 0, x, np.uint64(0) - x)
    x0 = orc.prg(64, 12, orc.tag("xs"), 0, n)
    xs = (x0, x - x0)
    ht = orc.hadamard_triplet_gen(13, 1, n)
    (r0, r1), _ = orc.secure_relu_fss(xs, orc.fss_dealer(14, 1, n), ht)
    (a0, a1), _ = orc.secure_relu(xs, orc.msb_dealer(15, 1, n), ht)
    assert np.array_equal(r0 + r1, a0 + a1)
    assert np.array_equal(r0 + r1, np.where(_signed(x, 64) >= 0, x, np.uint64(0)).astype(np.uint64))


@pytest.mark.parametrize("task,steps,tol_log2", [("logreg", 30, -16), ("mlp", 4, -15)])
def test_training_with_fss_comparison_tracks_fp64(task, steps, tol_log2):
    """The protocol with every ReLU / Eq. 9 comparison done by the one-round FSS DReLU (R22):
    decoded master weights vs fp64 SGD, and zero comparison mismatches / truncation failures."""
    import synth
    from oracle import plain
    from oracle import protocol as P
    Wi = synth.init_weights(task)
    m, pm = P.Model(task, Wi, compare="fss"), plain.PlainModel(task, Wi)
    P.diag_reset(True)
    try:
        for s in range(steps):
            X, Y = synth.batch(task, s)
            P.train_step(m, X, Y, s)
            pm.step(X, Y)
        d = dict(P.DIAG)
    finally:
        P.diag_reset(False)
    assert d["msb_checked"] > 0 and d["msb_fail"] == 0 and d["trunc_fail"] == 0, d
    err = max(np.abs(a - b).max() for a, b in zip(m.decoded_master(), pm.W))
    assert err < 2.0 ** tol_log2, np.log2(err)
