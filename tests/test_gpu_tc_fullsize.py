"""Config 5 at its full size in the launch configuration bench.py times (gpu): 4096^3 and
8192^3 ring GEMMs on tcgen05, checked on sampled output entries computed one by one by the
oracle (Python big-int dot products of the sampled row/column), plus Freivalds' check
C r == A (B r) mod 2^l with the oracle's ring matmul for random r (K = 8192 vector work)."""
import numpy as np
import pytest
import torch

from oracle import bruteforce as bf
from tests.util import to_dev, to_np

pytestmark = pytest.mark.gpu
SEED = 0x50534D4C


@pytest.mark.parametrize("n,l", [(4096, 64), (4096, 32), (8192, 64)])
def test_config5_fullsize_sampled_and_freivalds(orc, n, l):
    from paper_conf_icpp_chenzzzz020_b200 import build, psml
    build.build()
    ctx = psml.Ctx(l=l, backend=0)   # auto = tcgen05 at these sizes, as bench.py runs it
    A = psml.prg_fill(ctx.ring, 1, psml.tag("bA"), 0, n * n).view(n, n)
    B = psml.prg_fill(ctx.ring, 1, psml.tag("bB"), 0, n * n).view(n, n)
    C = psml.ring_gemm(ctx, A, B)
    torch.cuda.synchronize()
    rng = np.random.default_rng(n + l)
    rows = rng.integers(0, n, 6)
    cols = rng.integers(0, n, 6)
    iv = (lambda t: t.view(torch.int64)) if l == 64 else (lambda t: t.view(torch.int32))  # noqa: E731
    m = np.uint64((1 << l) - 1)
    a_rows = iv(A)[torch.from_numpy(rows).cuda()].cpu().numpy().astype(np.uint64) & m
    b_cols = iv(B)[:, torch.from_numpy(cols).cuda()].cpu().numpy().astype(np.uint64) & m
    c = to_np(C)
    for i, r in enumerate(rows):
        for j, cc in enumerate(cols):
            want = sum(int(x) * int(y) for x, y in zip(a_rows[i], b_cols[:, j])) % (1 << l)
            assert int(c[r, cc]) == want, (r, cc)
    # Freivalds: C r == A (B r) (mod 2^l), two random vectors
    for t in range(2):
        rv = orc.prg(l, SEED, orc.tag("fr"), t, n).reshape(n, 1)
        Br = orc.ring_matmul(to_np(B), rv, l)
        ABr = orc.ring_matmul(to_np(A), Br, l)
        Cr = orc.ring_matmul(c, rv, l)
        assert np.array_equal(ABr, Cr)
    ctx.close()
