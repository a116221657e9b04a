"""A few pipelined-graph MLP training steps (for `ncu` launch lists of the graph's kernels)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
from paper_conf_icpp_chenzzzz020_b200.train import SecureTrainer

task = sys.argv[1] if len(sys.argv) > 1 else "mlp"
steps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
tr = SecureTrainer(task, synth.init_weights(task))
X, Y = synth.batch(task, 0)
X, Y = torch.from_numpy(X).cuda(), torch.from_numpy(Y).cuda()
tr.step(X, Y, 0)
tr.capture(pipelined=True)
for s in range(1, steps + 1):
    tr.graph_step(X, Y, s)
torch.cuda.synchronize()
print("done")
