"""tcgen05 limb ring GEMM (backend 2) vs the oracle: bit-exact in Z_2^64 and Z_2^32 (gpu).

Covers single and multiple tiles, ragged M/N/K tails (zero-padded limb planes), split-K with
atomic partials, the l = 64 exactness limit (K' > 16512 forces exact chunks; all-ones operands
are the worst case for the int32 shift accumulators), the dealer's Z = U.V and the Beaver
product with its fused open + Z_i + truncation epilogue.  Each ring runs twice: on the limb-plane
kernels (psml_options.tc_small = 0) and on the in-kernel limb-split kernel (tc_small = 2; l = 64
wherever K' <= 16384, l = 32 always; one-segment plain products, cluster split-K over the GPU).
"""
import numpy as np
import pytest

from tests.util import pair_dev, pair_np, to_dev, to_np

pytestmark = pytest.mark.gpu
SEED = 0x50534D4C


@pytest.fixture(scope="module")
def P():
    from paper_conf_icpp_chenzzzz020_b200 import build, psml
    build.build()
    return psml


@pytest.fixture(scope="module", params=[(64, 0), (64, 2), (32, 0), (32, 2)],
                ids=["l64-planes", "l64-split", "l32-planes", "l32-split"])
def tctx(P, request):
    l, small = request.param
    c = P.Ctx(l=l, frac_bits=13, backend=2, options={"tc_small": small})
    yield c
    c.close()


def _rand(orc, l, n, salt):
    return orc.prg(l, SEED, orc.tag("tT"), salt, n)


@pytest.mark.parametrize("shape", [(128, 32, 64), (128, 64, 128), (1, 1, 1), (130, 33, 65),
                                   (256, 100, 130), (300, 777, 200), (512, 512, 512),
                                   (128, 4000, 64), (1000, 96, 1000), (640, 2048, 384), (2048, 1024, 2048)])
def test_tc_ring_gemm_bitexact(P, orc, tctx, shape):
    l = tctx.l
    M, K, N = shape
    a = _rand(orc, l, M * K, M + 7 * K).reshape(M, K)
    b = _rand(orc, l, K * N, N + 3 * K).reshape(K, N)
    C = P.ring_gemm(tctx, to_dev(a, l), to_dev(b, l))
    want = orc.ring_matmul(a, b, l)
    got = to_np(C)
    if not np.array_equal(got, want):
        bad = np.argwhere(got != want)
        raise AssertionError(f"{len(bad)} mismatches, first at {bad[:5].tolist()}: "
                             f"got {got[tuple(bad[0])]} want {want[tuple(bad[0])]}")


@pytest.mark.parametrize("K", [16384, 16512, 20000])
def test_tc_all_ones_exactness_limit(P, tctx, K):
    l = tctx.l
    ones = (1 << l) - 1
    A = to_dev(np.full((128, K), ones, np.uint64), l)
    B = to_dev(np.full((K, 64), ones, np.uint64), l)
    C = P.ring_gemm(tctx, A, B)
    assert np.all(to_np(C) == K % (1 << l))


@pytest.mark.parametrize("shape", [(128, 64, 128), (300, 130, 260)])
def test_tc_triplet_gen(P, orc, tctx, shape):
    M, K, N = shape
    U, V, Z = P.triplet_gen(tctx, SEED + 2, 4242, M, K, N)
    want = orc.triplet_gen(SEED + 2, 4242, M, K, N, tctx.l)
    for g, w in zip(pair_np(U) + pair_np(V) + pair_np(Z), want):
        assert np.array_equal(g, w)


@pytest.mark.parametrize("shape,flags", [((128, 64, 128), 0), ((256, 200, 192), 0), ((300, 130, 260), 3),
                                         ((512, 784, 128), 1), ((128, 9000, 64), 0), ((1024, 1000, 1100), 2)])
def test_tc_beaver_matmul_bitexact(P, orc, tctx, shape, flags):
    l = tctx.l
    M, K, N = shape
    a = _rand(orc, l, M * K, 1).reshape((K, M) if flags & 1 else (M, K))
    b = _rand(orc, l, K * N, 2).reshape((N, K) if flags & 2 else (K, N))
    A, B = orc.share(a, SEED + 1, 1, l), orc.share(b, SEED + 1, 2, l)
    trip = orc.triplet_gen(SEED + 2, 3, M, K, N, l)
    opA = [np.ascontiguousarray(t.T) if flags & 1 else t for t in A]
    opB = [np.ascontiguousarray(t.T) if flags & 2 else t for t in B]
    W0, W1 = orc.beaver_matmul(opA, opB, trip, trunc=13, l=l)
    td = [to_dev(t, l) for t in trip]
    C = P.secure_matmul(tctx, pair_dev(A, l), pair_dev(B, l), td[0:2], td[2:4], td[4:6], M, K, N,
                        flags=flags, trunc=13)
    assert np.array_equal(to_np(C[0]), W0) and np.array_equal(to_np(C[1]), W1)
