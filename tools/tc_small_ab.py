"""A/B of psml_options.tc_small on config-5 shapes: plain ring GEMM and co-resident Beaver matmul
in Z_2^l on tcgen05, limb-plane kernels (0) vs the in-kernel limb-split kernel (2).

    python tools/tc_small_ab.py [n1,n2,...] [64,32]    # one JSON line per (n, l, tc_small)
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_icpp_chenzzzz020_b200 import psml  # noqa: E402


def tev(fn, reps):
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    fn()
    ts = []
    for _ in range(reps):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda._sleep(200_000)   # ~0.1 ms of GPU work: the host submits fn() meanwhile, so the
        a.record()                   # events bracket device time, not host launch latency
        fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return sorted(ts)[len(ts) // 2]


ns = [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "256,512,1024,2048,4096").split(",")]
ls = [int(x) for x in (sys.argv[2] if len(sys.argv) > 2 else "64").split(",")]
for n, l in [(n, l) for l in ls for n in ns]:
    pairs = 36 if l == 64 else 10
    ring = psml.Ring(l, 13)
    A = psml.prg_fill(ring, 1, psml.tag("bA"), 0, n * n).view(n, n)
    B = psml.prg_fill(ring, 1, psml.tag("bB"), 0, n * n).view(n, n)
    res = {}
    for small in (0, 2):
        ctx = psml.Ctx(l=l, backend=2, options={"tc_small": small})
        C = psml.empty(0, l, (n, n))
        ms = tev(lambda: psml.ring_gemm(ctx, A, B, out=C), 10)
        res[small] = C.clone()
        As = psml.share(ring, 7, 1, A)
        Bs = psml.share(ring, 7, 2, B)
        U, V, Z = psml.triplet_gen(ctx, 3, 0, n, n, n)
        Cs = psml.empty_pair((n, n), l)
        bms = tev(lambda: psml.secure_matmul(ctx, As, Bs, U, V, Z, n, n, n, trunc=13, out=Cs), 10)
        res[(small, "b")] = [c.clone() for c in Cs]
        ctx.close()
        print(json.dumps({"n": n, "l": l, "tc_small": small, "plain_ms": ms,
                          "plain_tops": 2.0 * pairs * n ** 3 / ms / 1e9, "beaver_ms": bms,
                          "beaver_tops": 4 * 2.0 * pairs * n ** 3 / bms / 1e9}), flush=True)
    same = torch.equal(res[0], res[2]) and all(torch.equal(x, y) for x, y in zip(res[(0, "b")], res[(2, "b")]))
    print(json.dumps({"n": n, "l": l, "plain_and_beaver_identical": bool(same)}), flush=True)
