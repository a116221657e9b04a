"""CUPTI kernel durations (torch.profiler) of stand-alone psml calls, to separate device time from
launch gaps.  python tools/kernel_times.py [n1,n2,..] [tc_small]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
from torch.profiler import ProfilerActivity, profile  # noqa: E402

from paper_conf_icpp_chenzzzz020_b200 import psml  # noqa: E402

ns = [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "256,512,1024").split(",")]
small = int(sys.argv[2]) if len(sys.argv) > 2 else 2
for n in ns:
    ring = psml.Ring(64, 13)
    A = psml.prg_fill(ring, 1, psml.tag("bA"), 0, n * n).view(n, n)
    B = psml.prg_fill(ring, 1, psml.tag("bB"), 0, n * n).view(n, n)
    ctx = psml.Ctx(l=64, backend=2, options={"tc_small": small})
    C = psml.empty(0, 64, (n, n))
    As, Bs = psml.share(ring, 7, 1, A), psml.share(ring, 7, 2, B)
    U, V, Z = psml.triplet_gen(ctx, 3, 0, n, n, n)
    Cs = psml.empty_pair((n, n), 64)
    for _ in range(3):
        psml.ring_gemm(ctx, A, B, out=C)
        psml.secure_matmul(ctx, As, Bs, U, V, Z, n, n, n, trunc=13, out=Cs)
    torch.cuda.synchronize()
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        for _ in range(5):
            psml.ring_gemm(ctx, A, B, out=C)
            torch.cuda.synchronize()
        for _ in range(5):
            psml.ring_gemm(ctx, A, B, out=C)
        torch.cuda.synchronize()
        for _ in range(10):
            psml.secure_matmul(ctx, As, Bs, U, V, Z, n, n, n, trunc=13, out=Cs)
        torch.cuda.synchronize()
    ev = sorted([e for e in prof.events() if e.device_type == torch.autograd.DeviceType.CUDA],
                key=lambda e: e.time_range.start)
    print(f"n={n} tc_small={small}")
    t_prev = None
    for e in ev[:40]:
        gap = (e.time_range.start - t_prev) if t_prev is not None else 0
        print(f"   {e.name[:60]:60s} dur {e.time_range.elapsed_us():8.1f} us  gap {gap:8.1f}")
        t_prev = e.time_range.end
    ctx.close()
