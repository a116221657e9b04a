import sys, os
sys.path.insert(0, os.getcwd())
import torch
from paper_conf_icpp_chenzzzz020_b200 import psml
for n in (256, 512, 1024):
    ring = psml.Ring(64, 13)
    A = psml.prg_fill(ring, 1, psml.tag("bA"), 0, n * n).view(n, n)
    B = psml.prg_fill(ring, 1, psml.tag("bB"), 0, n * n).view(n, n)
    ctx = psml.Ctx(l=64, backend=2, options={"tc_small": 2})
    C = psml.empty(0, 64, (n, n))
    for r in range(3):
        print("=== n", n, "rep", r, flush=True)
        psml.ring_gemm(ctx, A, B, out=C); torch.cuda.synchronize()
