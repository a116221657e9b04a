"""CUPTI kernel durations of the MLP step's dealer alone (psml_model_deal, synchronised calls)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
from torch.profiler import ProfilerActivity, profile  # noqa: E402

import synth  # noqa: E402
from paper_conf_icpp_chenzzzz020_b200.train import SecureTrainer  # noqa: E402

task = sys.argv[1] if len(sys.argv) > 1 else "mlp"
tr = SecureTrainer(task, synth.init_weights(task))
for s in range(3):
    tr.deal(s)
torch.cuda.synchronize()
with profile(activities=[ProfilerActivity.CUDA]) as prof:
    for s in range(3, 8):
        tr.deal(s)
        torch.cuda.synchronize()
ev = sorted([e for e in prof.events() if e.device_type == torch.autograd.DeviceType.CUDA], key=lambda e: e.time_range.start)
t0 = None
for e in ev:
    if t0 is None or e.time_range.start - t0 > 500:
        t0 = e.time_range.start
        print("--- deal call")
    print(f"  +{e.time_range.start - t0:7.1f} dur {e.time_range.elapsed_us():7.1f} us  {e.name[:90]}")
