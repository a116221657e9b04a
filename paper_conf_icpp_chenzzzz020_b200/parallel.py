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


def strong_rows(pair, n_pairs, global_batch):
    """Rows of a global minibatch trained by pair `pair` of `n_pairs` under strong scaling
    (R28): [pair b, (pair + 1) b) with b = global_batch / n_pairs, a multiple
    of 8 (the row-sliced dealer streams start on ChaCha20 block boundaries)."""
    b = global_batch // n_pairs if n_pairs > 0 else 0
    if n_pairs <= 0 or b * n_pairs != global_batch or b % 8:
        raise ValueError(f"global batch {global_batch} does not split into {n_pairs} pairs of 8k rows")
    return slice(pair * b, (pair + 1) * b)


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


class CompressedChannel:
    """Compressed transmission of PAPER.md Sec. 4.4 (Eqs. 10-12) for the split deployment.

    Each message slot remembers the last message it sent and received.  The next message of the
    slot is sent as its delta against the previous one (E_{i,j+1} = E_{i,j} + Delta, Eq. 11), in
    CSR form when >= 75% of the delta is zero (psml_delta_encode) and dense otherwise; the receiver
    rebuilds the peer's message with psml_delta_apply.  The first message of a slot is dense.
    Two exchanges per compressed message: an 8-word header (format, nnz), then the payload.
    (With fresh masks per step the delta of a masked message is uniformly random -- dense; only a
    constant operand under a persistent mask gives an empty CSR, R19.)
    """

    def __init__(self, ctx, peer, group=None):
        self.ctx, self.peer, self.group = ctx, peer, group
        self.prev_send, self.prev_recv = {}, {}
        self.bytes_sent = 0
        self.formats = []

    def _words(self, t):
        return t.view(torch.int64) if t.dtype == torch.uint64 else t.view(torch.int32)

    def exchange(self, key, t):
        from . import psml
        if t.dim() != 2:
            raise ValueError("messages are matrices (rows x cols)")
        prev = self.prev_send.get(key)
        if prev is None:
            (r,) = exchange([t], self.peer, self.group)
            self.bytes_sent += t.numel() * t.element_size()
            self.formats.append("dense-first")
        else:
            enc = psml.delta_encode(self.ctx, t, prev)
            rows, cols = t.shape
            hdr = torch.tensor([1 if enc["is_csr"] else 0, enc["nnz"], rows, cols, 0, 0, 0, 0],
                               dtype=torch.int64, device=t.device)
            (phdr,) = exchange([hdr], self.peer, self.group)
            p_csr, p_nnz = int(phdr[0]), int(phdr[1])
            if enc["is_csr"]:
                send = [enc["row_ptr"]] + ([enc["col_idx"], enc["vals"]] if enc["nnz"] else [])
                self.bytes_sent += 64 + sum(x.numel() * x.element_size() for x in send)
            else:
                send = [enc["dense"]]
                self.bytes_sent += 64 + t.numel() * t.element_size()
            self.formats.append("csr" if enc["is_csr"] else "dense")
            # receive the peer's payload (shapes known from its header)
            if p_csr:
                recv_like = [torch.empty(rows + 1, dtype=torch.int32, device=t.device)]
                if p_nnz:
                    recv_like += [torch.empty(p_nnz, dtype=torch.int32, device=t.device),
                                  torch.empty(p_nnz, dtype=t.dtype, device=t.device)]
            else:
                recv_like = [torch.empty_like(t)]
            got = _exchange_uneven(send, recv_like, self.peer, self.group)
            r = self.prev_recv[key].clone()
            if p_csr:
                penc = dict(is_csr=True, nnz=p_nnz, row_ptr=got[0],
                            col_idx=got[1] if p_nnz else None, vals=got[2] if p_nnz else None)
            else:
                penc = dict(is_csr=False, nnz=p_nnz, dense=got[0])
            psml.delta_apply(self.ctx, r, penc)
        self.prev_send[key] = t.clone()
        self.prev_recv[key] = r.clone()
        return r


def _exchange_uneven(send, recv_like, peer, group=None):
    """Send the tensors `send` and receive tensors shaped like `recv_like` (may differ)."""
    import torch.distributed as dist
    stage = dist.get_backend(group) != "nccl"
    cast = lambda t: t.view(torch.int64) if t.dtype == torch.uint64 else (  # noqa: E731
        t.view(torch.int32) if t.dtype == torch.uint32 else t)
    ops, dst = [], []
    for t in send:
        src = cast(t)
        ops.append(dist.P2POp(dist.isend, src.cpu() if stage else src, peer, group))
    for t in recv_like:
        d = torch.empty_like(cast(t), device="cpu") if stage else torch.empty_like(cast(t))
        ops.append(dist.P2POp(dist.irecv, d, peer, group))
        dst.append((t, d))
    for req in dist.batch_isend_irecv(ops):
        req.wait()
    return [(d.to(t.device) if stage else d).view(t.dtype) for t, d in dst]


def split_secure_matmul_compressed(ctx, channel, slot, party, A_i, B_i, U_i, V_i, Z_i, M, K, N,
                                   flags=0, trunc=0):
    """split_secure_matmul with the opening sent through a CompressedChannel (slot = message id)."""
    from . import psml
    E, F = psml.beaver_mask(ctx, party, A_i, B_i, U_i, V_i, M, K, N, flags)
    Er = channel.exchange((slot, "E"), E)
    Fr = channel.exchange((slot, "F"), F)
    return psml.beaver_open_matmul(ctx, party, E, Er, F, Fr, U_i, V_i, Z_i, M, K, N, trunc)


# ---------------------------------------------------------------------------------------------
# Transports of the split training step (psml_party_forward_backward): every opening round of
# the step is one symmetric exchange between the two parties of a pair.
# ---------------------------------------------------------------------------------------------
def pair_layout(world):
    """Split deployment over `world` ranks: pair k = (rank k = party 0, rank k + world/2 =
    party 1).  Returns a function rank -> (party, pair, peer_rank)."""
    if world < 2 or world % 2:
        raise ValueError(f"the split deployment needs an even number of ranks, got {world}")
    half = world // 2

    def of(rank):
        party, pair = divmod(rank, half)
        return party, pair, (rank + half) % world
    return of


def host_staged_exchange_fn(peer, group=None):
    """A psml exchange callback that stages messages through host memory over any
    torch.distributed backend (gloo): sync the device, D2H, send/recv, H2D, sync."""
    import torch.distributed as dist
    from . import psml

    def fn(msgs, _stream):
        torch.cuda.synchronize()
        ops, back = [], []
        for send, recv, nbytes in msgs:
            if nbytes == 0:
                continue
            src = psml.wrap_bytes(send, nbytes).cpu()
            dst = torch.empty(nbytes, dtype=torch.uint8)
            ops.append(dist.P2POp(dist.isend, src, peer, group))
            ops.append(dist.P2POp(dist.irecv, dst, peer, group))
            back.append((recv, nbytes, dst, src))
        for req in dist.batch_isend_irecv(ops):
            req.wait()
        for recv, nbytes, dst, _ in back:
            psml.wrap_bytes(recv, nbytes).copy_(dst)
        torch.cuda.synchronize()
    return fn


def _swap_bytes(blob, party, peer, group=None):
    """Exchange a small byte blob with the peer rank over the process group (party 0 sends
    first; device tensors on nccl, host tensors otherwise)."""
    import torch.distributed as dist
    dev = "cuda" if dist.get_backend(group) == "nccl" else "cpu"
    mine = torch.frombuffer(bytearray(blob), dtype=torch.uint8).to(dev)
    theirs = torch.empty_like(mine)
    if party == 0:
        dist.send(mine, peer, group)
        dist.recv(theirs, peer, group)
    else:
        dist.recv(theirs, peer, group)
        dist.send(mine, peer, group)
    return bytes(theirs.cpu().numpy().tobytes())


def make_transport(party, peer, group=None, kind="peer", capacity_bytes=64 << 20):
    """The pair transport of the split deployment (include/psml.h):
      peer      (default) library peer-memory mailboxes mapped over CUDA IPC -- NVLink P2P stores
                between GPUs, shared HBM for two processes on one GPU; one kernel per exchange,
                graph-capturable; the process group only ships the 256-byte handles once;
      nccl      a library-owned 2-rank NCCL communicator (send/recv per exchange);
      callback  host-staged exchange over the process group (any backend, not capturable)."""
    import torch.distributed as dist
    from . import psml
    if kind == "peer":
        xp, blob = psml.Transport.peer(party, capacity_bytes)
        ok = 1
        try:
            xp.connect(_swap_bytes(blob, party, peer, group))
        except psml.PsmlError:   # e.g. no peer access between the two GPUs: both sides fall back
            ok = 0
        ok_peer = int.from_bytes(_swap_bytes(bytes([ok]), party, peer, group), "little")
        if ok and ok_peer:
            return xp
        xp.close()
        import sys
        print("psml: peer-memory transport unavailable between the pair's GPUs; using NCCL send/recv",
              file=sys.stderr)
        kind = "nccl"
    if kind == "nccl":
        uid = psml.nccl_unique_id() if party == 0 else bytes(128)
        got = _swap_bytes(uid, party, peer, group)
        return psml.Transport.nccl(uid if party == 0 else got, party)
    if kind == "callback":
        return psml.Transport.callback(host_staged_exchange_fn(peer, group))
    raise ValueError(kind)


def make_dp(ranks, rank, group=None):
    """The library-owned data-parallel communicator of one party over its global `ranks`
    (psml_dp_create): the first rank of the party creates the NCCL unique id and broadcasts it
    over `group` (a torch.distributed group holding exactly `ranks`)."""
    import torch.distributed as dist
    from . import psml
    size = len(ranks)
    me = ranks.index(rank)
    if size == 1:
        return psml.DataParallel(None, 0, 1)
    dev = "cuda" if dist.get_backend(group) == "nccl" else "cpu"
    uid = torch.zeros(128, dtype=torch.uint8, device=dev)
    if me == 0:
        uid.copy_(torch.frombuffer(bytearray(psml.nccl_unique_id()), dtype=torch.uint8))
    dist.broadcast(uid, ranks[0], group)
    return psml.DataParallel(bytes(uid.cpu().numpy().tobytes()), me, size)
