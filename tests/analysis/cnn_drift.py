"""Per-layer drift of the secure CNN vs fp64 SGD over one epoch (diagnostic; test-side analysis, so it may use oracle/)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, torch
import synth
from oracle import plain
from paper_conf_icpp_chenzzzz020_b200.train import SecureTrainer
task = "cnn"
Wi = synth.init_weights(task)
tr = SecureTrainer(task, Wi)
pm = plain.PlainModel(task, Wi)
X, Y = synth.batch(task, 0)
tr.step(torch.from_numpy(X), torch.from_numpy(Y), 0); pm.step(X, Y)
tr.capture(pipelined=True)
for s in range(1, 390):
    X, Y = synth.batch(task, s)
    tr.graph_step(torch.from_numpy(X), torch.from_numpy(Y), s); pm.step(X, Y)
    if s in (10, 50, 100, 200, 389):
        got = [w.cpu().numpy() for w in tr.master_weights()]
        errs = [np.abs(g.reshape(w.shape) - w) for g, w in zip(got, pm.W)]
        print(s, " ".join(f"L{i}: max 2^{np.log2(e.max()):.2f} p99.9 2^{np.log2(np.quantile(e, 0.999)):.2f} |w|max {np.abs(pm.W[i]).max():.3f}" for i, e in enumerate(errs)), flush=True)
