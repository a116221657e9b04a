"""GPU time per secure_matmul on the MLP shapes, per backend, from the library's CUDA events."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_icpp_chenzzzz020_b200 import psml

SHAPES = [(128, 784, 128, 0), (128, 128, 128, 0), (128, 128, 10, 0), (128, 10, 128, 2),
          (128, 128, 128, 1), (784, 128, 128, 1), (128, 3072, 64, 0), (12544, 128, 64, 1),
          (128, 64, 12544, 2), (1024, 1024, 1024, 0)]

def run(be, M, K, N, f, reps=20):
    ctx = psml.Ctx(backend=be)
    A = psml.empty_pair((K, M) if f & 1 else (M, K), 64)
    B = psml.empty_pair((N, K) if f & 2 else (K, N), 64)
    for x in A + B: x.zero_()
    U, V, Z = psml.triplet_gen(ctx, 1, 2, M, K, N)
    C = psml.empty_pair((M, N), 64)
    psml.secure_matmul(ctx, A, B, U, V, Z, M, K, N, flags=f, trunc=13, out=C)
    torch.cuda.synchronize()
    tot = 0.0
    for cls in (psml.PROF_GEMM, psml.PROF_TC, psml.PROF_MASK):
        psml.prof_enable(cls); psml.prof_read()
        for _ in range(reps):
            psml.secure_matmul(ctx, A, B, U, V, Z, M, K, N, flags=f, trunc=13, out=C)
        ms, n, w = psml.prof_read()
        tot += ms / reps * 1e3
    psml.prof_enable(-1)
    ctx.close()
    return tot

for (M, K, N, f) in SHAPES:
    r = {be: run(be, M, K, N, f) for be in (1, 2)}
    print(json.dumps(dict(M=M, K=K, N=N, flags=f, simt_us=r[1], tc_us=r[2])), flush=True)
