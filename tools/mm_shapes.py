"""Time psml_secure_matmul (both parties) on the MLP step's shapes for each GEMM backend."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_icpp_chenzzzz020_b200 import psml

SHAPES = [(128, 784, 128, 0), (128, 128, 128, 0), (128, 128, 10, 0), (128, 128, 10, 1),
          (128, 10, 128, 2), (128, 128, 128, 1), (784, 128, 128, 1), (4096, 4096, 4096, 0)]

def t(ctx, M, K, N, flags, reps=20):
    l = 64
    A = psml.empty_pair((K, M) if flags & 1 else (M, K), l)
    B = psml.empty_pair((N, K) if flags & 2 else (K, N), l)
    for x in A + B: x.zero_()
    U, V, Z = psml.triplet_gen(ctx, 1, 2, M, K, N)
    C = psml.empty_pair((M, N), l)
    psml.secure_matmul(ctx, A, B, U, V, Z, M, K, N, flags=flags, trunc=13, out=C)
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    r = reps if M * N * K < 1e9 else 3
    a.record()
    for _ in range(r):
        psml.secure_matmul(ctx, A, B, U, V, Z, M, K, N, flags=flags, trunc=13, out=C)
    b.record(); torch.cuda.synchronize()
    return a.elapsed_time(b) / r * 1e3

for be in (1, 2):
    ctx = psml.Ctx(backend=be)
    for (M, K, N, f) in SHAPES:
        us = t(ctx, M, K, N, f)
        print(json.dumps(dict(backend=be, M=M, K=K, N=N, flags=f, us=us,
                              ring_tmacs=2 * 2 * M * K * N / us / 1e6)), flush=True)
    ctx.close()
