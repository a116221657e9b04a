"""Per-phase globaltimer breakdown of tc_seg_kernel inside MLP training steps (TCSEG_TIMING build).

    PSML_NVCC_EXTRA=-DTCSEG_TIMING python -m paper_conf_icpp_chenzzzz020_b200.build --force
    python tools/tcseg_timing.py [steps]      # kernel printf lines on stdout
Then rebuild without the flag.  Eager steps, so each product runs without a concurrent dealer.
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_icpp_chenzzzz020_b200.train import SecureTrainer  # noqa: E402

steps = int(sys.argv[1]) if len(sys.argv) > 1 else 3
tr = SecureTrainer("mlp", synth.init_weights("mlp"))
for s in range(steps):
    X, Y = synth.batch("mlp", s)
    tr.deal(s)
    torch.cuda.synchronize()
    print(f"=== step {s}", flush=True)
    Xs, Ys = tr.share_batch(torch.from_numpy(X), torch.from_numpy(Y), s)
    tr.step_shares(Xs, Ys, s, deal=False)
    torch.cuda.synchronize()
