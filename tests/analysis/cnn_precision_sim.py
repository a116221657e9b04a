"""Statistical model of the secure CNN's fixed-point noise vs fp64 SGD (diagnostic only).

Replaces every SecureML share truncation (R7) by stochastic rounding -- the
distribution it realises (floor or floor + 1 with P(+1) = frac) -- and runs one CIFAR-shaped
epoch (390 steps of 128) for several forward-weight precisions f_w per layer (R21):
  W = trunc(W^m, m - f_w);  z = trunc(h . W, f_w);  delta_prev = trunc(delta . W^T, f_w) (.) DReLU.
Prints max |W^m - W_fp64| per layer.  Usage: python tests/analysis/cnn_precision_sim.py [steps]
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np  # noqa: E402

import synth  # noqa: E402

F, LR, M = 13, 14, 27
rng = np.random.default_rng(1)


def sr(x, f):
    y = x * 2.0 ** f
    fl = np.floor(y)
    return (fl + (rng.random(y.shape) < (y - fl))) / 2.0 ** f


def q(x, f):
    return np.rint(x * 2.0 ** f) / 2.0 ** f


def conv(X, W, k=5):
    """Direct valid conv: X (B,C,H,W), W ((c,ky,kx), o) -> (B,OH,OW,o)."""
    B, C, H, Wd = X.shape
    OH, OW = H - k + 1, Wd - k + 1
    Wr = W.reshape(C, k, k, -1)
    out = np.zeros((B, OH, OW, W.shape[1]))
    for ky in range(k):
        for kx in range(k):
            out += np.einsum("bchw,co->bhwo", X[:, :, ky:ky + OH, kx:kx + OW], Wr[:, ky, kx, :])
    return out


def conv_gw(X, D, k=5):
    B, C, H, Wd = X.shape
    OH, OW = H - k + 1, Wd - k + 1
    g = np.zeros((C, k, k, D.shape[-1]))
    for ky in range(k):
        for kx in range(k):
            g[:, ky, kx, :] = np.einsum("bchw,bhwo->co", X[:, :, ky:ky + OH, kx:kx + OW], D)
    return g.reshape(C * k * k, -1)


def run(fw, steps, secure):
    W = [q(w, M) for w in synth.init_weights("cnn")]
    for s in range(steps):
        X, Y = synth.batch("cnn", s)
        X, Y = q(X, F), q(Y, F)
        B = X.shape[0]
        X4 = X.reshape(B, 3, 32, 32)
        Wf = [sr(w, fw[i]) if secure else w for i, w in enumerate(W)]
        t = (lambda v, f: sr(v, F)) if secure else (lambda v, f: v)
        zc = t(conv(X4, Wf[0]), fw[0])
        m0 = zc >= 0
        h1 = np.maximum(zc, 0).reshape(B, -1)
        z2 = t(h1 @ Wf[1], fw[1])
        m1 = z2 >= 0
        h2 = np.maximum(z2, 0)
        yhat = np.clip(t(h2 @ Wf[2], fw[2]) + 0.5, 0, 1)
        d = yhat - Y
        g2 = h2.T @ d
        d = t(d @ Wf[2].T, fw[2]) * m1
        g1 = h1.T @ d
        d = (t(d @ Wf[1].T, fw[1]) * m0.reshape(B, -1)).reshape(B, 28, 28, 16)
        g0 = conv_gw(X4, d)
        for i, g in enumerate((g0, g1, g2)):
            upd = g * 2.0 ** -LR
            W[i] = W[i] - (sr(upd, M) if secure else upd)
    return W


if __name__ == "__main__":
    steps = int(sys.argv[1]) if len(sys.argv) > 1 else 390
    configs = [tuple(int(v) for v in a.split(",")) for a in sys.argv[2:]] or [(13, 13, 13), (13, 20, 20)]
    ref = run((F, F, F), steps, secure=False)
    for fw in configs:
        got = run(fw, steps, secure=True)
        errs = [np.abs(a - b).max() for a, b in zip(got, ref)]
        print("f_w", fw, " ".join(f"L{i} 2^{np.log2(e):.2f}" for i, e in enumerate(errs)),
              f"max 2^{np.log2(max(errs)):.2f}", flush=True)
