"""Test helpers: numpy <-> torch device transfers for ring tensors (no method arithmetic)."""
import numpy as np
import torch


def to_np(t):
    """Device ring tensor -> numpy uint64 (l = 32 values widened, high bits zero)."""
    a = t.detach().cpu().numpy()
    return a.astype(np.uint64)


def to_dev(a, l=64):
    dt = np.uint64 if l == 64 else np.uint32
    return torch.from_numpy(np.ascontiguousarray(np.asarray(a).astype(dt))).cuda()


def pair_np(p):
    return to_np(p[0]), to_np(p[1])


def pair_dev(p, l=64):
    return to_dev(p[0], l), to_dev(p[1], l)
