"""Plaintext float64 training -- the reference for BASELINE north_star's weight pin
("decoded floating-point model weights within 2^-12 absolute of a plaintext fp64 reference after
one epoch").  TEST INFRASTRUCTURE ONLY.

Same model, loss gradient and schedule as oracle/protocol.py (R10, R13-R15), but in
ordinary float64 with no ring, no shares and no truncation:
  linear   yhat = X w;            logistic yhat = f(X w) with PAPER.md Eq. 9 f(x) = clamp(x+1/2, 0, 1)
  MLP/CNN  ReLU hidden layers, Eq. 9 output, delta = yhat - y (derivative of Eq. 9 not applied)
  SGD      W -= (eta / |B|) X^T delta with eta / |B| = 2^-14
It starts from the decoded initial master weights and sees the decoded (13-bit) inputs, so the
only differences from the secure run are fixed-point rounding and truncation noise.
"""
import numpy as np

from .protocol import F, LR_SHIFT, MASTER, CNN_GEOM, WD_SHIFT, RNN_GEOM


def q(x, f):
    """Round to the fixed-point grid the client encodes on (independent of the ring)."""
    return np.rint(np.asarray(x, dtype=np.float64) * 2.0 ** f) / 2.0 ** f


def eq9(x):
    return np.clip(x + 0.5, 0.0, 1.0)


def conv2d(X4, W, k):
    """Direct valid stride-1 convolution (cross-correlation), written from its definition and
    independent of core.im2col:  out[b, oy, ox, o] = sum_{c,ky,kx} X[b, c, oy+ky, ox+kx] *
    W[(c, ky, kx), o].  X4: (B, C, H, W); W: (C*k*k, Cout) with rows ordered (c, ky, kx)."""
    B, C, H, Wd = X4.shape
    OH, OW = H - k + 1, Wd - k + 1
    Wr = W.reshape(C, k, k, -1)
    out = np.zeros((B, OH, OW, W.shape[1]), dtype=np.result_type(X4, W))
    for ky in range(k):
        for kx in range(k):
            out += np.einsum("bchw,co->bhwo", X4[:, :, ky:ky + OH, kx:kx + OW], Wr[:, ky, kx, :])
    return out


def conv2d_grad_w(X4, D, k):
    """dL/dW of conv2d: g[(c, ky, kx), o] = sum_{b,oy,ox} X[b, c, oy+ky, ox+kx] * D[b, oy, ox, o]."""
    B, C, H, Wd = X4.shape
    OH, OW = H - k + 1, Wd - k + 1
    g = np.zeros((C, k, k, D.shape[-1]), dtype=np.result_type(X4, D))
    for ky in range(k):
        for kx in range(k):
            g[:, ky, kx, :] = np.einsum("bchw,bhwo->co", X4[:, :, ky:ky + OH, kx:kx + OW], D)
    return g.reshape(C * k * k, -1)


class PlainModel:
    def __init__(self, task, W_init):
        self.task = task
        self.W = [q(W, MASTER) for W in W_init]

    def forward(self, X):
        if self.task in ("linreg", "svm"):
            return [X], [], X @ self.W[0]
        if self.task == "logreg":
            return [X], [], eq9(X @ self.W[0])
        if self.task == "mlp":
            acts, masks, h = [X], [], X
            for W in self.W[:-1]:
                z = h @ W
                masks.append(z >= 0)
                h = np.maximum(z, 0.0)
                acts.append(h)
            return acts, masks, eq9(h @ self.W[-1])
        if self.task == "cnn":
            g = CNN_GEOM
            B = X.shape[0]
            X4 = X.reshape(B, g["C"], g["H"], g["W"])
            zc = conv2d(X4, self.W[0], g["k"])               # (B, OH, OW, Cout)
            m0 = zc >= 0
            h1 = np.maximum(zc, 0.0).reshape(B, -1)          # rows (b), cols (oy, ox, o)
            z2 = h1 @ self.W[1]
            m1 = z2 >= 0
            h2 = np.maximum(z2, 0.0)
            return [X4, h1, h2], [m0.reshape(B, -1), m1], eq9(h2 @ self.W[2])
        raise ValueError(self.task)

    def step(self, X, Y):
        X, Y = q(X, F), q(Y, F)
        if self.task == "rnn":   # backpropagation through time (R25)
            return self._rnn_step(X, Y)
        acts, masks, yhat = self.forward(X)
        if self.task == "svm":   # hinge subgradient + weight decay (R24)
            delta = -Y * ((Y * yhat) < 1.0)
            g = X.T @ delta
            self.W[0] = self.W[0] - 2.0 ** -LR_SHIFT * g - 2.0 ** -WD_SHIFT * self.W[0]
            return yhat
        delta = yhat - Y
        lr = 2.0 ** -LR_SHIFT
        grads = [None] * len(self.W)
        for layer in range(len(self.W) - 1, -1, -1):
            a = acts[layer]
            if self.task == "cnn" and layer == 0:
                g = CNN_GEOM
                OH, OW = g["H"] - g["k"] + 1, g["W"] - g["k"] + 1
                grads[0] = conv2d_grad_w(a, delta.reshape(-1, OH, OW, g["Cout"]), g["k"])
                continue
            grads[layer] = a.T @ delta
            if layer > 0:
                delta = (delta @ self.W[layer].T) * masks[layer - 1]
        for layer, gr in enumerate(grads):
            self.W[layer] = self.W[layer] - lr * gr
        return yhat

    def _rnn_step(self, X, Y):
        g = RNN_GEOM
        T, D, H = g["T"], g["D"], g["H"]
        W1, Wo = self.W
        h = np.zeros((X.shape[0], H))
        As, masks = [], []
        for t in range(T):
            A = np.concatenate([X[:, t * D:(t + 1) * D], h], axis=1)
            z = A @ W1
            As.append(A)
            masks.append(z >= 0)
            h = np.maximum(z, 0.0)
        yhat = eq9(h @ Wo)
        delta = yhat - Y
        gWo = h.T @ delta
        delta = (delta @ Wo.T) * masks[T - 1]
        gW1 = np.zeros_like(W1)
        for t in range(T - 1, -1, -1):
            gW1 += As[t].T @ delta
            if t > 0:
                delta = (delta @ W1[D:, :].T) * masks[t - 1]
        lr = 2.0 ** -LR_SHIFT
        self.W = [W1 - lr * gW1, Wo - lr * gWo]
        return yhat
