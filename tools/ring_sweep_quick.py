"""Quick ring-GEMM timing (config 5 sizes) for A/B builds: python tools/ring_sweep_quick.py [n ...]."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_icpp_chenzzzz020_b200 import psml  # noqa: E402

ns = [int(a) for a in sys.argv[1:]] or [512, 1024, 2048]
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for n in ns:
    for l in [int(x) for x in os.environ.get("RING_LS", "64,32").split(",")]:
        ctx = psml.Ctx(l=l, backend=2)
        A = psml.prg_fill(ctx.ring, 1, psml.tag("bA"), 0, n * n).view(n, n)
        B = psml.prg_fill(ctx.ring, 1, psml.tag("bB"), 0, n * n).view(n, n)
        C = psml.empty(0, l, (n, n))
        psml.ring_gemm(ctx, A, B, out=C)
        ts = []
        for _ in range(9):
            flush.zero_()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda._sleep(200_000)   # device busy while the host submits: events bracket device time
            a.record()
            psml.ring_gemm(ctx, A, B, out=C)
            b.record()
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        ms = sorted(ts)[4]
        pairs = 36 if l == 64 else 10
        print(f"n={n} l={l} ms={ms:.4f} TOPS={pairs * 2 * n ** 3 / ms / 1e9:.0f}", flush=True)
        ctx.close()
