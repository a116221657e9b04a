"""GPU parity of every hot-path primitive against the CPU oracle, through the C ABI (gpu).

Bar: bit-exact (integer ring arithmetic) for every share, opened value and dealer word, on the
same seeded inputs; sizes span several tiles and a ragged tail; l = 32 and 64.
"""
import glob
import json
import os

import numpy as np
import pytest
import torch

from oracle import bruteforce as bf
from tests.util import pair_dev, pair_np, to_dev, to_np

pytestmark = pytest.mark.gpu
SEED = 0x50534D4C
GOLDEN = sorted(glob.glob(os.path.join(os.path.dirname(__file__), "golden", "beaver_l*.json")))


@pytest.fixture(scope="module")
def P():
    from paper_conf_icpp_chenzzzz020_b200 import build, psml
    build.build()
    return psml


@pytest.fixture(scope="module", params=[64, 32])
def ctx(P, request):
    c = P.Ctx(l=request.param, frac_bits=13, backend=1)
    yield c
    c.close()


def _rand(orc, l, n, salt):
    return orc.prg(l, SEED, orc.tag("tR"), salt, n)


# --- client side -------------------------------------------------------------------------------
@pytest.mark.parametrize("l", [64, 32])
@pytest.mark.parametrize("n,offset", [(1, 0), (13, 5), (1000, 0), (4099, 77), (1 << 20, 3)])
def test_prg_fill(P, orc, l, n, offset):
    g = P.prg_fill(P.Ring(l, 13), 0xDEADBEEF, orc.tag("U1"), 0x0102030405060708, n, offset=offset)
    torch.cuda.synchronize()
    want = orc.prg(l, 0xDEADBEEF, orc.tag("U1"), 0x0102030405060708, n, offset=offset)
    assert np.array_equal(to_np(g), want)


@pytest.mark.parametrize("l", [64, 32])
def test_encode_decode_share_reconstruct(P, orc, l):
    ring = P.Ring(l, 13)
    rng = np.random.default_rng(3)
    x = np.concatenate([rng.normal(0, 3, 5000), [0.5 / 8192, 1.5 / 8192, -2.5 / 8192, 0.0, -1.0]])
    v = P.encode(ring, torch.from_numpy(x))
    want = orc.encode(x, l, 13)
    assert np.array_equal(to_np(v), want)
    back = P.decode(ring, v).cpu().numpy()
    assert np.array_equal(back, orc.decode(want, l, 13))
    x0, x1 = P.share(ring, SEED + 1, 42, v)
    w0, w1 = orc.share(want, SEED + 1, 42, l)
    assert np.array_equal(to_np(x0), w0) and np.array_equal(to_np(x1), w1)
    assert np.array_equal(to_np(P.reconstruct(ring, x0, x1)), want)
    # fused client pass (psml_encode_share) == encode then share, on ragged sizes
    for n in (1, 7, 17, len(x)):
        xs = torch.from_numpy(x[:n]).cuda()
        y0, y1 = P.encode_share(ring, SEED + 1, 43, xs)
        u0, u1 = orc.share(orc.encode(x[:n], l, 13), SEED + 1, 43, l)
        assert np.array_equal(to_np(y0), u0) and np.array_equal(to_np(y1), u1), n


@pytest.mark.parametrize("l", [64, 32])
def test_encode_share_from_pixels_and_class_indices(P, orc, l):
    """psml_encode_share_u8 (x = q / 255 from 8-bit pixels) and psml_encode_share_onehot (one-hot
    labels from class indices) equal the oracle's encode + share of the float64 batch, on the
    synthetic MNIST/CIFAR batches and on ragged sizes, every pixel value 0..255 included."""
    import synth
    ring = P.Ring(l, 13)
    for task in ("mlp", "cnn"):
        X, Y = synth.batch(task, 5)
        q, cls = synth.batch_u8(task, 5)
        x0, x1 = P.encode_share_u8(ring, SEED + 1, 44, torch.from_numpy(q).cuda())
        w0, w1 = orc.share(orc.encode(X.reshape(-1), l, 13), SEED + 1, 44, l)
        assert np.array_equal(to_np(x0).reshape(-1), w0) and np.array_equal(to_np(x1).reshape(-1), w1), task
        y0, y1 = P.encode_share_onehot(ring, SEED + 1, 45, torch.from_numpy(cls).cuda(), 10)
        v0, v1 = orc.share(orc.encode(Y.reshape(-1), l, 13), SEED + 1, 45, l)
        assert np.array_equal(to_np(y0).reshape(-1), v0) and np.array_equal(to_np(y1).reshape(-1), v1), task
    q = np.arange(256, dtype=np.uint8)
    for n in (1, 9, 256):
        x0, x1 = P.encode_share_u8(ring, SEED + 1, 46, torch.from_numpy(q[:n]).cuda())
        w0, w1 = orc.share(orc.encode(q[:n].astype(np.float64) / 255.0, l, 13), SEED + 1, 46, l)
        assert np.array_equal(to_np(x0), w0) and np.array_equal(to_np(x1), w1), n


@pytest.mark.parametrize("l", [64, 32])
def test_truncate(P, orc, l):
    ring = P.Ring(l, 13)
    x = _rand(orc, l, 10007, 1)
    for party in (0, 1):
        for d in (1, 13, 27):
            t = to_dev(x, l)
            P.truncate(ring, party, t, d)
            assert np.array_equal(to_np(t), orc.truncate(x, party, d, l))


# --- dealer ------------------------------------------------------------------------------------
@pytest.mark.parametrize("shape", [(4, 4, 4), (3, 5, 2), (130, 67, 70), (128, 784, 1), (65, 300, 129)])
def test_triplet_gen(P, orc, ctx, shape):
    M, K, N = shape
    U, V, Z = P.triplet_gen(ctx, SEED + 2, 777, M, K, N)
    want = orc.triplet_gen(SEED + 2, 777, M, K, N, ctx.l)
    got = pair_np(U) + pair_np(V) + pair_np(Z)
    for g, w in zip(got, want):
        assert np.array_equal(g, w)


@pytest.mark.parametrize("M_total,cuts,K,N", [(100, (0, 37, 100), 33, 65), (4096, (0, 1024, 2048, 3072, 4096), 16, 8),
                                               (9, (0, 1, 9), 1, 1)])
def test_triplet_gen_rows_are_slices_of_the_full_triplet(P, orc, ctx, M_total, cuts, K, N):
    """psml_triplet_gen_rows (M-row sharding, R28): row blocks (ragged, unaligned to
    ChaCha20 blocks) equal the oracle's full triplet sliced; V is the whole V of every block."""
    want = orc.triplet_gen(SEED + 2, 4242, M_total, K, N, ctx.l)
    for r0, r1 in zip(cuts[:-1], cuts[1:]):
        U, V, Z = P.triplet_gen_rows(ctx, SEED + 2, 4242, M_total, r0, r1 - r0, K, N)
        got = pair_np(U) + pair_np(V) + pair_np(Z)
        rows = slice(r0, r1)
        for g, w, sliced in zip(got, want, (True, True, False, False, True, True)):
            assert np.array_equal(g, w[rows] if sliced else w)
    with pytest.raises(P.PsmlError):
        P.triplet_gen_rows(ctx, SEED + 2, 4242, M_total, M_total - 1, 2, K, N)


def test_hadamard_triplet_and_msb_material(P, orc, ctx):
    ring = ctx.ring
    for n in (1, 17, 5003):
        U, V, Z = P.hadamard_triplet_gen(ring, SEED + 2, 99, n)
        want = orc.hadamard_triplet_gen(SEED + 2, 99, n, ctx.l)
        for g, w in zip(pair_np(U) + pair_np(V) + pair_np(Z), want):
            assert np.array_equal(g, w)
        m = P.msb_dealer(ring, SEED + 2, 123, n)
        w0, w1 = orc.msb_dealer(SEED + 2, 123, n, ctx.l)
        assert np.array_equal(to_np(m[0]), w0) and np.array_equal(to_np(m[1]), w1)


# --- Beaver matmul -----------------------------------------------------------------------------
SHAPES = [(4, 4, 4), (3, 5, 2), (128, 784, 1), (784, 128, 1), (128, 784, 128), (128, 128, 10),
          (784, 128, 128), (100, 37, 65), (257, 129, 200), (64, 3000, 64), (130, 8192, 66),
          (1, 16, 1), (129, 33, 65)]


@pytest.mark.parametrize("shape", SHAPES)
@pytest.mark.parametrize("flags", [0, 1, 2, 3])
def test_secure_matmul_bitexact(P, orc, ctx, shape, flags):
    l = ctx.l
    M, K, N = shape
    a = _rand(orc, l, M * K, 10 + M).reshape((K, M) if flags & 1 else (M, K))
    b = _rand(orc, l, K * N, 20 + N).reshape((N, K) if flags & 2 else (K, N))
    A = orc.share(a, SEED + 1, 1, l)
    B = orc.share(b, SEED + 1, 2, l)
    trip = orc.triplet_gen(SEED + 2, 3, M, K, N, l)
    opA = [np.ascontiguousarray(t.T) if flags & 1 else t for t in A]
    opB = [np.ascontiguousarray(t.T) if flags & 2 else t for t in B]
    trunc = 13 if (M * K) % 2 else 0
    (W0, W1), tr = orc.beaver_matmul(opA, opB, trip, trunc=trunc, l=l, trace=True)
    td = [to_dev(t, l) for t in trip]
    C, T = P.secure_matmul(ctx, pair_dev(A, l), pair_dev(B, l), td[0:2], td[2:4], td[4:6], M, K, N,
                           flags=flags, trunc=trunc, trace=True)
    torch.cuda.synchronize()
    assert np.array_equal(to_np(C[0]), W0) and np.array_equal(to_np(C[1]), W1)
    for k in ("E0", "E1", "E", "F0", "F1", "F"):
        assert np.array_equal(to_np(T[k]), tr[k]), k


@pytest.mark.parametrize("shape", [(128, 784, 1), (784, 128, 1), (1, 16, 1), (3, 5, 1), (300, 2049, 1)])
@pytest.mark.parametrize("trunc", [0, 13])
def test_secure_matmul_gemv_single_launch(P, orc, ctx, shape, trunc):
    """Config 1 (N = 1, untraced): the mask, open and GEMV rounds fused into one launch
    (beaver_gemv_kernel) -- bit-exact vs the oracle."""
    l = ctx.l
    M, K, N = shape
    a = _rand(orc, l, M * K, 30 + M).reshape(M, K)
    b = _rand(orc, l, K * N, 40 + K).reshape(K, N)
    A, B = orc.share(a, SEED + 1, 3, l), orc.share(b, SEED + 1, 4, l)
    trip = orc.triplet_gen(SEED + 2, 5, M, K, N, l)
    W0, W1 = orc.beaver_matmul(A, B, trip, trunc=trunc, l=l)
    td = [to_dev(t, l) for t in trip]
    n0 = P.kernel_launch_count()
    C = P.secure_matmul(ctx, pair_dev(A, l), pair_dev(B, l), td[0:2], td[2:4], td[4:6], M, K, N, trunc=trunc)
    torch.cuda.synchronize()
    assert P.kernel_launch_count() - n0 == 1
    assert np.array_equal(to_np(C[0]), W0) and np.array_equal(to_np(C[1]), W1)


@pytest.mark.parametrize("shape", [(4, 4, 4), (33, 70, 19), (128, 784, 128)])
def test_secure_matmul_paper_form(P, orc, ctx, shape):
    l = ctx.l
    M, K, N = shape
    A = orc.share(_rand(orc, l, M * K, 5).reshape(M, K), SEED + 1, 1, l)
    B = orc.share(_rand(orc, l, K * N, 6).reshape(K, N), SEED + 1, 2, l)
    trip = orc.triplet_gen(SEED + 2, 3, M, K, N, l)
    W0, W1 = orc.beaver_matmul(A, B, trip, form=1, l=l)
    td = [to_dev(t, l) for t in trip]
    C = P.secure_matmul(ctx, pair_dev(A, l), pair_dev(B, l), td[0:2], td[2:4], td[4:6], M, K, N,
                        flags=P.PAPER_FORM)
    assert np.array_equal(to_np(C[0]), W0) and np.array_equal(to_np(C[1]), W1)


@pytest.mark.parametrize("path", GOLDEN, ids=[os.path.basename(p) for p in GOLDEN])
def test_golden_worked_examples(P, path):
    d = json.load(open(path))
    l = d["l"]
    if l not in (32, 64):
        pytest.skip("GPU rings are l = 32, 64")
    c = P.Ctx(l=l, backend=1)
    a = lambda k: to_dev(np.array(d[k], dtype=np.uint64), l)  # noqa: E731
    M, K, N = d["M"], d["K"], d["N"]
    C, T = P.secure_matmul(c, (a("A0"), a("A1")), (a("B0"), a("B1")), (a("U0"), a("U1")),
                           (a("V0"), a("V1")), (a("Z0"), a("Z1")), M, K, N, trace=True)
    assert to_np(C[0]).tolist() == d["C0"] and to_np(C[1]).tolist() == d["C1"]
    for k in ("E0", "E1", "E", "F0", "F1", "F"):
        assert to_np(T[k]).tolist() == d[k]
    C = P.secure_matmul(c, (a("A0"), a("A1")), (a("B0"), a("B1")), (a("U0"), a("U1")),
                        (a("V0"), a("V1")), (a("Z0"), a("Z1")), M, K, N, trunc=d["trunc"])
    assert to_np(C[0]).tolist() == d["T0"] and to_np(C[1]).tolist() == d["T1"]
    c.close()


# --- elementwise protocol ------------------------------------------------------------------------
@pytest.mark.parametrize("n", [1, 31, 4097, 200003])
def test_secure_hadamard(P, orc, ctx, n):
    l = ctx.l
    A = orc.share(_rand(orc, l, n, 1), SEED + 1, 5, l)
    B = orc.share(_rand(orc, l, n, 2), SEED + 1, 6, l)
    trip = orc.hadamard_triplet_gen(SEED + 2, 7, n, l)
    W0, W1 = orc.beaver_hadamard(A, B, trip, l)
    td = [to_dev(t, l) for t in trip]
    C = P.secure_hadamard(ctx, pair_dev(A, l), pair_dev(B, l), td[0:2], td[2:4], td[4:6])
    assert np.array_equal(to_np(C[0]), W0) and np.array_equal(to_np(C[1]), W1)


def _edge_values(orc, l, n):
    top = 1 << l
    edges = [0, 1, 2, (top >> 1) - 1, top >> 1, top - 1, 4096, top - 4096, 8192, top - 8192]
    v = _rand(orc, l, n, 9)
    k = min(n, len(edges))
    v[:k] = np.array(edges[:k], dtype=np.uint64)
    return v


@pytest.mark.parametrize("n", [1, 10, 1000, 65537])
def test_secure_msb_relu_eq9(P, orc, ctx, n):
    l = ctx.l
    x = _edge_values(orc, l, n)
    X = orc.share(x, SEED + 1, 8, l)
    Xd = pair_dev(X, l)
    mat = orc.msb_dealer(SEED + 2, 11, n, l)
    matd = pair_dev(mat, l)
    (a0, a1), (b0, b1) = orc.secure_msb(X, mat, l, want_bool=True)
    ga, gb = P.secure_msb(ctx, Xd, matd, want_bool=True)
    assert np.array_equal(to_np(ga[0]), a0) and np.array_equal(to_np(ga[1]), a1)
    assert np.array_equal(to_np(gb[0]), b0) and np.array_equal(to_np(gb[1]), b1)
    assert np.array_equal(orc.reconstruct(to_np(ga[0]), to_np(ga[1]), l), x >> np.uint64(l - 1))
    ht = orc.hadamard_triplet_gen(SEED + 2, 12, n, l)
    (r0, r1), (d0, d1) = orc.secure_relu(X, mat, ht, l)
    htd = [to_dev(t, l) for t in ht]
    y, dr = P.secure_relu(ctx, Xd, matd, htd[0:2], htd[2:4], htd[4:6])
    assert np.array_equal(to_np(y[0]), r0) and np.array_equal(to_np(y[1]), r1)
    assert np.array_equal(to_np(dr[0]), d0) and np.array_equal(to_np(dr[1]), d1)
    mat2 = orc.msb_dealer(SEED + 2, 13, 2 * n, l)
    ht2 = orc.hadamard_triplet_gen(SEED + 2, 14, 2 * n, l)
    e0, e1 = orc.secure_eq9(X, mat2, ht2, l, 13)
    h2 = [to_dev(t, l) for t in ht2]
    ey = P.secure_eq9(ctx, Xd, pair_dev(mat2, l), h2[0:2], h2[2:4], h2[4:6])
    assert np.array_equal(to_np(ey[0]), e0) and np.array_equal(to_np(ey[1]), e1)
    # and the reconstruction is Eq. 9 on the grid (away from wrap-around)
    yv = orc.reconstruct(to_np(ey[0]), to_np(ey[1]), l)
    for v, got in list(zip(x, yv))[:2000]:
        s = bf.signed(int(v), l)
        if abs(s) < (1 << (l - 2)):
            assert int(got) == bf.eq9_fixed(int(v), l, 13)


# --- plain ring GEMM (config 5 kernel) ------------------------------------------------------------
@pytest.mark.parametrize("shape", [(1, 1, 1), (64, 64, 64), (100, 257, 130), (512, 512, 512)])
def test_ring_gemm(P, orc, ctx, shape):
    l = ctx.l
    M, K, N = shape
    a = _rand(orc, l, M * K, 31).reshape(M, K)
    b = _rand(orc, l, K * N, 32).reshape(K, N)
    C = P.ring_gemm(ctx, to_dev(a, l), to_dev(b, l))
    assert np.array_equal(to_np(C), orc.ring_matmul(a, b, l))


def test_ring_gemm_all_ones_worst_case(P, ctx):
    l = ctx.l
    K = 16384
    ones = (1 << l) - 1
    A = to_dev(np.full((128, K), ones, np.uint64), l)
    B = to_dev(np.full((K, 128), ones, np.uint64), l)
    C = P.ring_gemm(ctx, A, B)
    assert np.all(to_np(C) == K % (1 << l))   # K (2^l - 1)^2 = K mod 2^l


# --- compressed transmission ------------------------------------------------------------------------
@pytest.mark.parametrize("frac_changed", [0.0, 0.1, 0.25, 0.26, 1.0])
def test_delta_codec(P, orc, ctx, frac_changed):
    l = ctx.l
    rows, cols = 96, 130
    rng = np.random.default_rng(int(frac_changed * 100))
    prev = _rand(orc, l, rows * cols, 41).reshape(rows, cols)
    cur = prev.copy()
    k = int(round(frac_changed * rows * cols))
    idx = rng.choice(rows * cols, k, replace=False)
    cur.reshape(-1)[idx] = (cur.reshape(-1)[idx] + np.uint64(977)) & orc.mask(l)
    want = orc.delta_csr_encode(cur, prev, l)
    got = P.delta_encode(ctx, to_dev(cur, l), to_dev(prev, l))
    assert got["is_csr"] == want["is_csr"] and got["nnz"] == want["nnz"]
    if want["is_csr"]:
        assert np.array_equal(got["row_ptr"].cpu().numpy(), want["row_ptr"])
        assert np.array_equal(got["col_idx"].cpu().numpy(), want["col_idx"])
        assert np.array_equal(to_np(got["vals"]), want["vals"])
    else:
        assert np.array_equal(to_np(got["dense"]), want["dense"])
    t = to_dev(prev, l)
    P.delta_apply(ctx, t, got)
    assert np.array_equal(to_np(t), cur)


def test_msb_chain_per_round_kernels_match():
    """The one-kernel-per-round chain (split-deployment structure) gives the same shares as the
    cooperative single-launch chain: rerun the activation parity tests with PSML_MSB_CHAIN=rounds."""
    import subprocess
    import sys
    env = dict(os.environ, PSML_MSB_CHAIN="rounds")
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-m", "gpu", "-k",
                        "test_secure_msb_relu_eq9", __file__], env=env, capture_output=True, text=True,
                       cwd=os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-2000:]
