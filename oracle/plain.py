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

from . import core
from .protocol import F, LR_SHIFT, MASTER, CNN_GEOM


def q(x, f):
    """Round to the fixed-point grid the client encodes on (independent of the ring)."""
    return np.rint(np.asarray(x, dtype=np.float64) * 2.0 ** f) / 2.0 ** f


def eq9(x):
    return np.clip(x + 0.5, 0.0, 1.0)


class PlainModel:
    def __init__(self, task, W_init):
        self.task = task
        self.W = [q(W, MASTER) for W in W_init]

    def forward(self, X):
        if self.task == "linreg":
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
            P = core.im2col(X, g["C"], g["H"], g["W"], g["k"])
            zc = P @ self.W[0]
            m0 = zc >= 0
            h1 = np.maximum(zc, 0.0).reshape(B, -1)
            z2 = h1 @ self.W[1]
            m1 = z2 >= 0
            h2 = np.maximum(z2, 0.0)
            return [P, h1, h2], [m0.reshape(B, -1), m1], eq9(h2 @ self.W[2])
        raise ValueError(self.task)

    def step(self, X, Y):
        X, Y = q(X, F), q(Y, F)
        acts, masks, yhat = self.forward(X)
        delta = yhat - Y
        lr = 2.0 ** -LR_SHIFT
        grads = [None] * len(self.W)
        for layer in range(len(self.W) - 1, -1, -1):
            a = acts[layer]
            if self.task == "cnn" and layer == 0:
                g = CNN_GEOM
                delta = delta.reshape(-1, g["Cout"])
            grads[layer] = a.T @ delta
            if layer > 0:
                delta = (delta @ self.W[layer].T) * masks[layer - 1]
        for layer, gr in enumerate(grads):
            self.W[layer] = self.W[layer] - lr * gr
        return yhat
