"""Kernel timeline of pipelined-graph training steps (CUPTI via torch.profiler, no serialisation).

    python tools/timeline.py [task] [steps] [out.json]

Prints, for the last few steps, every kernel's start offset / duration (us) relative to the step's
first kernel, its stream, and the union of busy time per stream, so the overlap of the dealer
branch (next step's material) with the online chain can be read off directly.
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_icpp_chenzzzz020_b200.train import SecureTrainer  # noqa: E402

task = sys.argv[1] if len(sys.argv) > 1 else "mlp"
steps = int(sys.argv[2]) if len(sys.argv) > 2 else 20
out = sys.argv[3] if len(sys.argv) > 3 else "gpurun_out/timeline.json"
tr = SecureTrainer(task, synth.init_weights(task))
X, Y = synth.batch(task, 0)
X, Y = torch.from_numpy(X).cuda(), torch.from_numpy(Y).cuda()
tr.step(X, Y, 0)
tr.capture(pipelined=True)
for s in range(1, 6):
    tr.graph_step(X, Y, s)
torch.cuda.synchronize()
from torch.profiler import ProfilerActivity, profile  # noqa: E402

with profile(activities=[ProfilerActivity.CUDA]) as prof:
    for s in range(6, 6 + steps):
        tr.graph_step(X, Y, s)
    torch.cuda.synchronize()
prof.export_chrome_trace(out)
ev = [e for e in json.load(open(out))["traceEvents"] if e.get("cat") == "kernel"]
ev.sort(key=lambda e: e["ts"])
# a step starts at each encode_share pair (client launches before each replay)
def _share(e):   # the client's share launch(es) open each step
    return "encode_share" in e["name"] or "client_share" in e["name"]


starts = [e["ts"] for i, e in enumerate(ev) if _share(e) and (i == 0 or not _share(ev[i - 1]))]
print(f"{len(ev)} kernels, {len(starts)} steps; mean step {(starts[-1] - starts[0]) / (len(starts) - 1):.1f} us")
for k in range(len(starts) - 3, len(starts) - 1):
    t0, t1 = starts[k], starts[k + 1]
    print(f"--- step window {k}: {t1 - t0:.1f} us")
    busy = {}
    for e in ev:
        if t0 <= e["ts"] < t1:
            st = e["args"].get("stream", "?")
            nm = e["name"].split("(")[0].replace("void ", "").replace("psml::", "")[:60]
            print(f"  {e['ts'] - t0:8.1f} {e['dur']:7.1f}  s{st:<4} {nm}")
            busy.setdefault(st, []).append((e["ts"], e["ts"] + e["dur"]))
    for st, iv in busy.items():
        iv.sort()
        tot, cur = 0.0, None
        for a, b in iv:
            if cur is None or a > cur[1]:
                if cur:
                    tot += cur[1] - cur[0]
                cur = [a, b]
            else:
                cur[1] = max(cur[1], b)
        tot += cur[1] - cur[0]
        print(f"  stream {st}: busy {tot:.1f} us")
