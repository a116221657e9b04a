"""One plain ring GEMM n^3 (config 5) for ncu captures: python tools/ring_gemm_once.py N L [reps]."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_icpp_chenzzzz020_b200 import psml  # noqa: E402

n, l = int(sys.argv[1]), int(sys.argv[2])
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 2
ctx = psml.Ctx(l=l, backend=2)
A = psml.prg_fill(ctx.ring, 1, psml.tag("bA"), 0, n * n).view(n, n)
B = psml.prg_fill(ctx.ring, 1, psml.tag("bB"), 0, n * n).view(n, n)
C = psml.empty(0, l, (n, n))
for _ in range(reps):
    psml.ring_gemm(ctx, A, B, out=C)
torch.cuda.synchronize()
print("ok", n, l)
