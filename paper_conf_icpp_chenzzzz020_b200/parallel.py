"""Data-parallel plumbing over torch.distributed (R16, §9).

One co-resident party pair per GPU trains on its own minibatch rows (weak scaling).  After the
local forward/backward, each pair holds untruncated weight-gradient shares (26 fractional bits,
both parties, one contiguous [2][P] uint64 buffer).  Summing them over pairs is plain addition in
Z_{2^64}, which is exactly a two's-complement int64 SUM all-reduce (NCCL or gloo wrap on
overflow).  Every pair then applies the same update with log2(pairs) extra truncation bits
(eta / |B| with |B| = 128 * pairs), so the replicated weight shares stay identical.
"""
import math

import torch


def ring_allreduce_(t, group=None):
    """In-place sum of ring shares across the process group (uint64 viewed as int64)."""
    import torch.distributed as dist
    if not dist.is_initialized() or dist.get_world_size(group) == 1:
        return t
    v = t.view(torch.int64) if t.dtype == torch.uint64 else t
    if v.dtype != torch.int64:
        raise TypeError("ring shares must be uint64 or int64 tensors")
    dist.all_reduce(v, op=dist.ReduceOp.SUM, group=group)
    return t


def dp_update_shift(world):
    """Extra truncation bits for `world` data-parallel pairs (must be a power of two)."""
    s = int(round(math.log2(world))) if world > 0 else -1
    if world <= 0 or (1 << s) != world:
        raise ValueError(f"data-parallel pair count must be a power of two, got {world}")
    return s


def pair_rows(step, pair, n_pairs, batch, n_rows):
    """First row of minibatch `step` for pair `pair` of `n_pairs` (matches synth.batch)."""
    return ((step * n_pairs + pair) * batch) % (n_rows - batch + 1)
