"""Warm, in-graph latency of one co-resident secure matmul (mask + GEMM) on the MLP shapes.

Captures R back-to-back psml_secure_matmul calls into a CUDA graph and times replays with CUDA
events (the way the training step runs them).  Usage: python tools/gemm_lat.py [backend]
"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_icpp_chenzzzz020_b200 import psml

SHAPES = [(128, 784, 128, 0), (128, 128, 128, 0), (128, 128, 10, 0), (128, 10, 128, 2),
          (128, 128, 128, 1), (784, 128, 128, 1), (128, 128, 10, 1)]
be = int(sys.argv[1]) if len(sys.argv) > 1 else 1
R = 20
ctx = psml.Ctx(backend=be)
out = {}
for (M, K, N, f) in SHAPES:
    A = psml.empty_pair((K, M) if f & 1 else (M, K), 64)
    B = psml.empty_pair((N, K) if f & 2 else (K, N), 64)
    for x in A + B: x.view(torch.int64).random_()
    U, V, Z = psml.triplet_gen(ctx, 1, 2, M, K, N)
    C = psml.empty_pair((M, N), 64)
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        psml.secure_matmul(ctx, A, B, U, V, Z, M, K, N, flags=f, trunc=13, out=C)
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            for _ in range(R):
                psml.secure_matmul(ctx, A, B, U, V, Z, M, K, N, flags=f, trunc=13, out=C)
        g.replay(); torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        for _ in range(10): g.replay()
        e1.record(s)
        torch.cuda.synchronize()
    out[f"{M}x{K}x{N}/{f}"] = round(e0.elapsed_time(e1) * 1e3 / (10 * R), 2)
print(json.dumps(dict(backend=be, simt=os.environ.get("PSML_SIMT", "cl"), us_per_matmul=out)))
