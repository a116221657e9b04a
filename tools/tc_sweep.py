"""Config-5 sweep: ring GEMM n^3 for l = 32/64, tcgen05 vs CUDA-core, CUDA-event timing."""
import json, sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_icpp_chenzzzz020_b200 import psml

def run(n, l, backend, reps=5):
    ctx = psml.Ctx(l=l, backend=backend)
    A = psml.prg_fill(ctx.ring, 1, psml.tag("bA"), 0, n * n).view(n, n)
    B = psml.prg_fill(ctx.ring, 1, psml.tag("bB"), 0, n * n).view(n, n)
    C = psml.empty(0, l, (n, n))
    psml.ring_gemm(ctx, A, B, out=C)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    ts = []
    for _ in range(reps):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); psml.ring_gemm(ctx, A, B, out=C); b.record(); torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    ms = sorted(ts)[len(ts) // 2]
    pairs = 36 if l == 64 else 10
    ctx.close()
    return dict(n=n, l=l, backend=backend, ms=ms, tops=pairs * 2.0 * n ** 3 / ms / 1e9)

out = []
for n in [int(x) for x in sys.argv[1].split(",")]:
    for l in (64, 32):
        for be in ([2, 1] if n <= 4096 else [2]):
            r = run(n, l, be); out.append(r); print(json.dumps(r), flush=True)
