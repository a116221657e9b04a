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


# ---------------------------------------------------------------------------------------------
# Split deployment: party 0 and party 1 in different processes (distinct GPUs over NVLink with
# NCCL, or any backend).  One opening = one symmetric exchange of masked messages (R5).
# ---------------------------------------------------------------------------------------------
def exchange(send, peer, group=None):
    """Send each tensor in `send` to `peer` and receive same-shaped tensors from it.

    NCCL moves device tensors directly (NVLink P2P); other backends (gloo) stage through host
    memory.  Returns the received tensors on the device of `send`.
    """
    import torch.distributed as dist
    backend = dist.get_backend(group)
    stage = backend != "nccl"
    out = []
    ops = []
    bufs = []
    for t in send:
        src = t.view(torch.int64) if t.dtype == torch.uint64 else t.view(torch.int32)
        src = src.cpu() if stage else src
        dst = torch.empty_like(src)
        ops.append(dist.P2POp(dist.isend, src, peer, group))
        ops.append(dist.P2POp(dist.irecv, dst, peer, group))
        bufs.append((t, dst))
    for req in dist.batch_isend_irecv(ops):
        req.wait()
    for t, dst in bufs:
        r = dst.to(t.device) if stage else dst
        out.append(r.view(t.dtype))
    return out


def split_secure_matmul(ctx, party, A_i, B_i, U_i, V_i, Z_i, M, K, N, flags=0, trunc=0, peer=None,
                        group=None):
    """Party `party`'s share of A.B with the opening done over torch.distributed:
    psml_beaver_mask -> exchange(E_i, F_i) -> psml_beaver_open_matmul (Eqs. 4-8)."""
    from . import psml
    peer = 1 - party if peer is None else peer
    E, F = psml.beaver_mask(ctx, party, A_i, B_i, U_i, V_i, M, K, N, flags)
    Er, Fr = exchange([E, F], peer, group)
    return psml.beaver_open_matmul(ctx, party, E, Er, F, Fr, U_i, V_i, Z_i, M, K, N, trunc)
