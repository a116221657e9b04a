"""Seeded synthetic plaintext inputs shared by the oracle, the tests and bench.py.

This module holds NONE of the method's arithmetic (no encoding, sharing, ring or protocol
step): it only produces float64 plaintext data, labels and initial weights with the shapes and
value distributions of the paper's workloads:

  * MNIST-shaped rows (28x28 pixels 0..255): 784 8-bit pixels k, about 81%
    zeros, non-zeros uniform on 1..255 (MNIST's ~19% ink density); features x = k / 255.
  * CIFAR-10-shaped rows (3x32x32): 3072 dense 8-bit pixels uniform on 0..255,
    x = k / 255.
  * the pixel bytes themselves (`batch_u8`): what a client holding the images sends; the float64
    features are exactly k / 255.0 (IEEE division), so both forms encode to the same ring words.
  * labels from fixed random teachers (linear, thresholded linear, 784-128-128-10 ReLU MLP,
    5x5/16-channel conv net), one-hot for the 10-class tasks.

Every 128-row block b is drawn from its own generator ``default_rng([seed, kind, b])``, so any
row range is reproducible without generating the rows before it (the bench only materialises
the steps it times; the parity tests slice the same rows).
"""
import functools

import numpy as np

DATA_SEED = 0x50534D4C          # "PSML"
INIT_SEED = DATA_SEED + 3
TEACHER_SEED = DATA_SEED + 4
BLOCK = 128

MNIST_FEATURES = 784
CIFAR_SHAPE = (3, 32, 32)
CIFAR_FEATURES = 3 * 32 * 32
# SYNTHETIC sequences for the RNN ("RNN does not apply to images, so we only use our
# generated dataset, SYNTHETIC"): T steps of D dense 8-bit features; R25.
RNN_T, RNN_D, RNN_H, RNN_C = 16, 32, 64, 10
SEQ_FEATURES = RNN_T * RNN_D

_KIND = {"mnist": 1, "cifar": 2, "seq": 3}


def _block_pixels(kind, b, seed):
    rng = np.random.default_rng([seed, _KIND[kind], b])
    if kind == "mnist":
        x = rng.random((BLOCK, MNIST_FEATURES))
        keep = rng.random((BLOCK, MNIST_FEATURES)) < 0.19
        k = np.minimum(np.floor(x * 255.0), 254.0).astype(np.uint8) + 1   # 1..255
        return np.where(keep, k, 0).astype(np.uint8)
    width = CIFAR_FEATURES if kind == "cifar" else SEQ_FEATURES
    return np.minimum(np.floor(rng.random((BLOCK, width)) * 256.0), 255.0).astype(np.uint8)


def pixels(kind, start, count, seed=DATA_SEED):
    """8-bit pixels of rows [start, start+count) of the synthetic dataset `kind`."""
    if count <= 0:
        width = {"mnist": MNIST_FEATURES, "cifar": CIFAR_FEATURES, "seq": SEQ_FEATURES}[kind]
        return np.zeros((0, width), dtype=np.uint8)
    b0, b1 = start // BLOCK, (start + count - 1) // BLOCK
    blocks = np.concatenate([_block_pixels(kind, b, seed) for b in range(b0, b1 + 1)], axis=0)
    off = start - b0 * BLOCK
    return blocks[off:off + count]


def rows(kind, start, count, seed=DATA_SEED):
    """Rows [start, start+count) of the synthetic dataset `kind` ('mnist' | 'cifar'): k / 255."""
    return pixels(kind, start, count, seed).astype(np.float64) / 255.0


# ---------------------------------------------------------------------------------------------
# teachers (label generators)
# ---------------------------------------------------------------------------------------------
def linear_teacher(d=MNIST_FEATURES, seed=TEACHER_SEED):
    return np.random.default_rng([seed, 1]).uniform(-0.05, 0.05, size=(d, 1))


@functools.lru_cache(maxsize=None)
def logistic_threshold(seed=TEACHER_SEED):
    """Median of X w* over the first 8192 MNIST-shaped rows (fixed, data-independent of step)."""
    w = linear_teacher(seed=seed)
    return float(np.median(rows("mnist", 0, 8192) @ w))


def mlp_teacher(dims=(784, 128, 128, 10), seed=TEACHER_SEED):
    rng = np.random.default_rng([seed, 3])
    return [rng.normal(0.0, 1.0, size=(a, b)) / np.sqrt(a) for a, b in zip(dims[:-1], dims[1:])]


def cnn_teacher(seed=TEACHER_SEED, cout=16, k=5, hidden=64, classes=10):
    rng = np.random.default_rng([seed, 4])
    c = CIFAR_SHAPE[0]
    oh = CIFAR_SHAPE[1] - k + 1
    return [rng.normal(0.0, 1.0, size=(c * k * k, cout)) / np.sqrt(c * k * k),
            rng.normal(0.0, 1.0, size=(oh * oh * cout, hidden)) / np.sqrt(oh * oh * cout),
            rng.normal(0.0, 1.0, size=(hidden, classes)) / np.sqrt(hidden)]


def rnn_teacher(seed=TEACHER_SEED):
    rng = np.random.default_rng([seed, 5])
    return [rng.normal(0.0, 1.0, size=(RNN_D + RNN_H, RNN_H)) / np.sqrt(RNN_D + RNN_H),
            rng.normal(0.0, 1.0, size=(RNN_H, RNN_C)) / np.sqrt(RNN_H)]


def _patches(X, k=5):
    """(B, 3072) -> (B*28*28, 75) patch matrix for the teacher conv (label generation only)."""
    B = X.shape[0]
    c, h, w = CIFAR_SHAPE
    oh, ow = h - k + 1, w - k + 1
    X4 = X.reshape(B, c, h, w)
    out = np.empty((B, oh, ow, c, k, k))
    for ky in range(k):
        for kx in range(k):
            out[:, :, :, :, ky, kx] = X4[:, :, ky:ky + oh, kx:kx + ow].transpose(0, 2, 3, 1)
    return out.reshape(B * oh * ow, c * k * k)


def _one_hot(scores):
    y = np.zeros_like(scores)
    y[np.arange(scores.shape[0]), np.argmax(scores, axis=1)] = 1.0
    return y


def labels(task, X):
    relu = lambda t: np.maximum(t, 0.0)   # noqa: E731  (teacher nets only)
    if task == "linreg":
        return X @ linear_teacher()
    if task == "logreg":
        return (X @ linear_teacher() > logistic_threshold()).astype(np.float64)
    if task == "svm":      # +-1 labels of the same linear teacher (R24)
        return np.where(X @ linear_teacher() > logistic_threshold(), 1.0, -1.0)
    if task == "mlp":
        W = mlp_teacher()
        return _one_hot(relu(relu(X @ W[0]) @ W[1]) @ W[2])
    if task == "cnn":
        Wc, W1, W2 = cnn_teacher()
        h = relu(_patches(X) @ Wc).reshape(X.shape[0], -1)
        return _one_hot(relu(h @ W1) @ W2)
    if task == "rnn":
        W1, Wo = rnn_teacher()
        h = np.zeros((X.shape[0], RNN_H))
        for t in range(RNN_T):
            h = relu(np.concatenate([X[:, t * RNN_D:(t + 1) * RNN_D], h], axis=1) @ W1)
        return _one_hot(h @ Wo)
    raise ValueError(task)


TASK_DATA = {"linreg": "mnist", "logreg": "mnist", "svm": "mnist", "mlp": "mnist", "cnn": "cifar", "rnn": "seq"}
TASK_ROWS = {"mnist": 60000, "cifar": 50000, "seq": 60000}


def batch(task, step, batch_size=BLOCK, pair=0, n_pairs=1, seed=DATA_SEED):
    """Minibatch `step` of `task` for data-parallel pair `pair` of `n_pairs` (weak scaling:
    each pair gets its own `batch_size` rows).  Returns float64 (X, Y)."""
    kind = TASK_DATA[task]
    start = ((step * n_pairs + pair) * batch_size) % (TASK_ROWS[kind] - batch_size + 1)
    X = rows(kind, start, batch_size, seed)
    return X, labels(task, X)


def batch_u8(task, step, batch_size=BLOCK, pair=0, n_pairs=1, seed=DATA_SEED):
    """The same minibatch as `batch` in the client's compact form: (pixels uint8, labels), labels
    as uint8 class indices for the one-hot tasks (mlp, cnn), else the float64 labels of `batch`.
    batch() == (pixels / 255.0, one_hot(classes)) exactly."""
    kind = TASK_DATA[task]
    start = ((step * n_pairs + pair) * batch_size) % (TASK_ROWS[kind] - batch_size + 1)
    q = pixels(kind, start, batch_size, seed)
    Y = labels(task, q.astype(np.float64) / 255.0)
    if task in ("mlp", "cnn", "rnn"):
        return q, np.argmax(Y, axis=1).astype(np.uint8)
    return q, Y


def init_weights(task, dims=None, seed=INIT_SEED):
    """Initial plaintext weights (R13): zeros for linear/logistic regression,
    U(+-1/sqrt(fan_in)) for the MLP and CNN."""
    if task in ("linreg", "logreg", "svm"):
        return [np.zeros((MNIST_FEATURES, 1))]
    if task == "mlp":
        dims = dims or (784, 128, 128, 10)
        shapes = list(zip(dims[:-1], dims[1:]))
    elif task == "cnn":
        shapes = [(75, 16), (12544, 64), (64, 10)]
    elif task == "rnn":
        shapes = [(RNN_D + RNN_H, RNN_H), (RNN_H, RNN_C)]
    else:
        raise ValueError(task)
    rng = np.random.default_rng([seed, 7])
    return [rng.uniform(-1.0, 1.0, size=s) / np.sqrt(s[0]) for s in shapes]
