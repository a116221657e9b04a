"""Split deployment (one party per process) vs the oracle, bit-exact (gpu).

Two processes -- party 0 and party 1 -- each own only their shares; the opening is a symmetric
exchange over torch.distributed (gloo here, staged through host memory, so both processes can
share the single test GPU; NCCL moves the same device buffers over NVLink on a multi-GPU box).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu
SEED = 0x50534D4C
CASES = [((128, 784, 1), 0, 1), ((257, 129, 200), 3, 1), ((512, 784, 256), 0, 2), ((300, 200, 130), 1, 2)]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _inputs(l, M, K, N, flags):
    from oracle import core as orc
    a = orc.prg(l, SEED, orc.tag("sA"), M, M * K).reshape((K, M) if flags & 1 else (M, K))
    b = orc.prg(l, SEED, orc.tag("sB"), N, K * N).reshape((N, K) if flags & 2 else (K, N))
    A, B = orc.share(a, SEED + 1, 1, l), orc.share(b, SEED + 1, 2, l)
    trip = orc.triplet_gen(SEED + 2, 3, M, K, N, l)
    return A, B, trip


def _party(rank, port, l, outdir):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    from paper_conf_icpp_chenzzzz020_b200 import psml
    from paper_conf_icpp_chenzzzz020_b200.parallel import split_secure_matmul
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=2)
    torch.cuda.set_device(0)
    dt = np.uint64 if l == 64 else np.uint32
    dev = lambda x: torch.from_numpy(np.ascontiguousarray(x.astype(dt))).cuda()  # noqa: E731
    for ci, ((M, K, N), flags, backend) in enumerate(CASES):
        A, B, trip = _inputs(l, M, K, N, flags)
        ctx = psml.Ctx(l=l, backend=backend)
        C = split_secure_matmul(ctx, rank, dev(A[rank]), dev(B[rank]), dev(trip[rank]), dev(trip[2 + rank]),
                                dev(trip[4 + rank]), M, K, N, flags=flags, trunc=13)
        np.save(os.path.join(outdir, f"c{ci}_{rank}.npy"), C.cpu().numpy().astype(np.uint64))
        ctx.close()
    dist.destroy_process_group()


def _party_ctx(rank, port, l, outdir):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    from paper_conf_icpp_chenzzzz020_b200 import psml
    from paper_conf_icpp_chenzzzz020_b200.parallel import make_transport
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=2)
    torch.cuda.set_device(0)
    dt = np.uint64 if l == 64 else np.uint32
    dev = lambda x: torch.from_numpy(np.ascontiguousarray(x.astype(dt))).cuda()  # noqa: E731
    xp = make_transport(rank, 1 - rank, kind="peer", capacity_bytes=4 << 20)
    for ci, ((M, K, N), flags, backend) in enumerate(CASES):
        A, B, trip = _inputs(l, M, K, N, flags)
        ctx = psml.Ctx(l=l, backend=backend, party=rank, xport=xp)
        C = psml.secure_matmul_party(ctx, dev(A[rank]), dev(B[rank]), dev(trip[rank]), dev(trip[2 + rank]),
                                     dev(trip[4 + rank]), M, K, N, flags=flags, trunc=13)
        np.save(os.path.join(outdir, f"c{ci}_{rank}.npy"), C.cpu().numpy().astype(np.uint64))
        ctx.close()
    xp.close()
    dist.destroy_process_group()


@pytest.mark.parametrize("l", [64, 32])
def test_per_party_ctx_secure_matmul(tmp_path, l):
    """psml_ctx_create_party + psml_secure_matmul_party (SURVEY §8(b) one-party collective call):
    the exchange goes through the library's peer-memory transport; bit-exact vs the oracle."""
    from oracle import core as orc
    mp.spawn(_party_ctx, args=(_free_port(), l, str(tmp_path)), nprocs=2, join=True)
    for ci, ((M, K, N), flags, _) in enumerate(CASES):
        A, B, trip = _inputs(l, M, K, N, flags)
        opA = [np.ascontiguousarray(t.T) if flags & 1 else t for t in A]
        opB = [np.ascontiguousarray(t.T) if flags & 2 else t for t in B]
        W = orc.beaver_matmul(opA, opB, trip, trunc=13, l=l)
        for p in range(2):
            assert np.array_equal(np.load(tmp_path / f"c{ci}_{p}.npy"), W[p]), (ci, p)


@pytest.mark.parametrize("l", [64, 32])
def test_split_deployment_matches_oracle(tmp_path, l):
    from oracle import core as orc
    mp.spawn(_party, args=(_free_port(), l, str(tmp_path)), nprocs=2, join=True)
    for ci, ((M, K, N), flags, _) in enumerate(CASES):
        A, B, trip = _inputs(l, M, K, N, flags)
        opA = [np.ascontiguousarray(t.T) if flags & 1 else t for t in A]
        opB = [np.ascontiguousarray(t.T) if flags & 2 else t for t in B]
        W = orc.beaver_matmul(opA, opB, trip, trunc=13, l=l)
        for p in range(2):
            assert np.array_equal(np.load(tmp_path / f"c{ci}_{p}.npy"), W[p]), (ci, p)


def _party_compressed(rank, port, outdir):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    from oracle import core as orc
    from paper_conf_icpp_chenzzzz020_b200 import psml
    from paper_conf_icpp_chenzzzz020_b200.parallel import CompressedChannel, split_secure_matmul_compressed
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=2)
    torch.cuda.set_device(0)
    dev = lambda x: torch.from_numpy(np.ascontiguousarray(x)).cuda()  # noqa: E731
    M, K, N = 128, 784, 16
    ctx = psml.Ctx(l=64, backend=1)
    ch = CompressedChannel(ctx, 1 - rank)
    # "epochs" over the same data matrix A with a PERSISTENT mask U_A (R19): E repeats exactly,
    # its delta is empty CSR; B changes every epoch with a fresh V: F goes dense.
    a = orc.prg(64, SEED, orc.tag("cA"), 0, M * K).reshape(M, K)
    A = orc.share(a, SEED + 1, 5, 64)
    for ep in range(3):
        b = orc.prg(64, SEED, orc.tag("cB"), ep, K * N).reshape(K, N)
        B = orc.share(b, SEED + 1, 6 + ep, 64)
        U0, U1, _, _, _, _ = orc.triplet_gen(SEED + 2, 100, M, K, N, 64)       # persistent U
        _, _, V0, V1, _, _ = orc.triplet_gen(SEED + 2, 200 + ep, M, K, N, 64)  # fresh V
        U, V = (U0, U1), (V0, V1)
        Z = orc.ring_matmul(U0 + U1, V0 + V1)
        Z0 = orc.prg(64, SEED, orc.tag("cZ"), ep, M * N).reshape(M, N)
        Zs = (Z0, Z - Z0)
        C = split_secure_matmul_compressed(ctx, ch, 0, rank, dev(A[rank]), dev(B[rank]), dev(U[rank]),
                                           dev(V[rank]), dev(Zs[rank]), M, K, N, trunc=13)
        W = orc.beaver_matmul(A, B, (U0, U1, V0, V1, Zs[0], Zs[1]), trunc=13)
        np.save(os.path.join(outdir, f"ok{ep}_{rank}.npy"), np.array([np.array_equal(C.cpu().numpy(), W[rank])]))
    np.save(os.path.join(outdir, f"fmt_{rank}.npy"), np.array(ch.formats))
    dist.destroy_process_group()


def test_split_compressed_transmission(tmp_path):
    """PAPER.md Eqs. 10-12 + L228: a persistent-mask operand is re-opened from an empty CSR delta,
    a changing operand from a dense delta; shares stay bit-exact vs the oracle."""
    mp.spawn(_party_compressed, args=(_free_port(), str(tmp_path)), nprocs=2, join=True)
    for r in range(2):
        for ep in range(3):
            assert bool(np.load(tmp_path / f"ok{ep}_{r}.npy")[0]), (r, ep)
        fmts = list(np.load(tmp_path / f"fmt_{r}.npy"))
        assert fmts == ["dense-first", "dense-first", "csr", "dense", "csr", "dense"], fmts


# ---------------------------------------------------------------------------------------------
# Split training step (psml_party_forward_backward): party 0 and party 1 in two processes, every
# opening (Beaver E/F, each AND round of the MSB chain, the B2A word, the Hadamard E/F) through the
# library's transport -- here the host-staged gloo callback.  Each party's master-weight share
# must equal the oracle's simulation of both parties (oracle/protocol.py) after every step.
# ---------------------------------------------------------------------------------------------
SPLIT_TASKS = [("linreg", 2), ("logreg", 2), ("mlp", 2), ("cnn", 1)]
FSS_TASKS = [("logreg", 2), ("mlp", 2)]
REUSE_TASKS = [("linreg", 2), ("mlp", 2)]


def _party_train(rank, port, outdir, kind, compare="a2b", mask_reuse=False):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import synth
    from paper_conf_icpp_chenzzzz020_b200.parallel import make_dp, make_transport
    from paper_conf_icpp_chenzzzz020_b200.train import PartyTrainer
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    if kind == "peer_rounds":           # one kernel + one exchange per round instead of the fused chain
        os.environ["PSML_SPLIT_FUSED"] = "0"
        kind = "peer"
    dist.init_process_group("gloo", rank=rank, world_size=2)
    torch.cuda.set_device(0)
    xp = make_transport(rank, 1 - rank, kind=kind)
    dp = make_dp([rank], rank)          # one pair: the party's data-parallel group is itself
    tasks = REUSE_TASKS if mask_reuse else (SPLIT_TASKS if compare == "a2b" else FSS_TASKS)
    for task, steps in tasks:
        tr = PartyTrainer(task, synth.init_weights(task), rank, xp, backend=1, dp=dp, compare=compare,
                          mask_reuse=mask_reuse)
        for s in range(steps):
            X, Y = synth.batch(task, s)
            tr.step(torch.from_numpy(X), torch.from_numpy(Y), s)
            torch.cuda.synchronize()
            for layer in range(tr.model.n_layers):
                np.save(os.path.join(outdir, f"{task}_s{s}_l{layer}_{rank}.npy"),
                        tr.my_master_share(layer).cpu().numpy())
        tr.close()
    sent, n_ex = xp.stats()
    np.save(os.path.join(outdir, f"xstats_{rank}.npy"), np.array([sent, n_ex]))
    xp.close()
    dp.close()
    dist.destroy_process_group()


def _check_against_oracle(tmp_path, tasks, compare="a2b", mask_reuse=False):
    import synth
    from oracle import protocol as OP
    for task, steps in tasks:
        om = OP.Model(task, synth.init_weights(task), compare=compare, mask_reuse=mask_reuse)
        for s in range(steps):
            X, Y = synth.batch(task, s)
            OP.train_step(om, X, Y, s)
            for layer in range(len(om.Wm)):
                for p in range(2):
                    got = np.load(tmp_path / f"{task}_s{s}_l{layer}_{p}.npy")
                    assert np.array_equal(got.reshape(om.Wm[layer][p].shape), om.Wm[layer][p]), \
                        (task, s, layer, p)


@pytest.mark.parametrize("kind", ["peer", "peer_rounds", "callback"])
def test_split_training_matches_oracle(tmp_path, kind):
    """Two party processes on the one test GPU.  kind=peer: every Beaver opening is the library's
    peer-memory exchange kernel over CUDA-IPC-mapped mailboxes and every activation ONE kernel with
    its rounds' exchanges fused over the peer window (split_fused.cuh); peer_rounds: one kernel + one
    exchange per activation round; callback: host-staged gloo.  Each party's master shares equal
    the oracle's."""
    mp.spawn(_party_train, args=(_free_port(), str(tmp_path), kind), nprocs=2, join=True)
    _check_against_oracle(tmp_path, SPLIT_TASKS)
    st = [np.load(tmp_path / f"xstats_{p}.npy") for p in range(2)]
    assert st[0][1] == st[1][1] > 0 and st[0][0] == st[1][0] > 0   # symmetric exchanges


def test_split_training_fss_comparison_matches_oracle(tmp_path):
    """The split step with the one-round FSS comparison (R22): per ReLU / Eq. 9 one exchange of
    x_i + r_i and one Hadamard E/F exchange instead of 9 rounds; bit-exact vs the oracle."""
    mp.spawn(_party_train, args=(_free_port(), str(tmp_path), "peer", "fss"), nprocs=2, join=True)
    _check_against_oracle(tmp_path, FSS_TASKS, compare="fss")
    st = [np.load(tmp_path / f"xstats_{p}.npy") for p in range(2)]
    assert st[0][1] == st[1][1] > 0


def test_split_training_mask_reuse_matches_oracle(tmp_path):
    """Mask reuse in the split engine (R26): the backward products open delta once per layer and
    reuse this party's stored forward openings; fewer exchanges and bytes, bit-exact vs the oracle."""
    mp.spawn(_party_train, args=(_free_port(), str(tmp_path), "peer", "a2b", True), nprocs=2, join=True)
    _check_against_oracle(tmp_path, REUSE_TASKS, mask_reuse=True)


GRAPH_TASKS = [("mlp", 4), ("logreg", 3)]


def _party_graph(rank, port, outdir):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import synth
    from paper_conf_icpp_chenzzzz020_b200.parallel import make_dp, make_transport
    from paper_conf_icpp_chenzzzz020_b200.train import PartyTrainer
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=2)
    torch.cuda.set_device(0)
    xp = make_transport(rank, 1 - rank, kind="peer")
    dp = make_dp([rank], rank)
    for task, steps in GRAPH_TASKS:
        tr = PartyTrainer(task, synth.init_weights(task), rank, xp, dp=dp)
        X, Y = synth.batch(task, 0)
        tr.step(torch.from_numpy(X), torch.from_numpy(Y), 0)       # eager first step
        tr.capture_party(pipelined=True)
        for s in range(steps):
            if s > 0:
                X, Y = synth.batch(task, s)
                X_i, Y_i = tr.share_batch(X, Y, s)
                tr.graph_step_party(X_i, Y_i, s)
            torch.cuda.synchronize()
            for layer in range(tr.model.n_layers):
                np.save(os.path.join(outdir, f"{task}_s{s}_l{layer}_{rank}.npy"),
                        tr.my_master_share(layer).cpu().numpy())
        tr.close()
    xp.close()
    dp.close()
    dist.destroy_process_group()


def test_split_step_cuda_graph_matches_oracle(tmp_path):
    """The split step captured into a CUDA graph (psml_party_capture_step, pipelined dealer, the
    peer-memory exchanges and the library data-parallel all-reduce inside the graph) replayed
    for steps 1..n-1 of two party processes: bit-exact vs the oracle after every step."""
    mp.spawn(_party_graph, args=(_free_port(), str(tmp_path)), nprocs=2, join=True)
    _check_against_oracle(tmp_path, GRAPH_TASKS)


# ---------------------------------------------------------------------------------------------
# Dealer key separation + compressed distribution (R23): a dealer/client process (this
# test) holds the dealer seed, deals every step and writes each party's bundle of derived words
# and its input / weight shares; the two party processes get only their own seed s_i, regenerate
# their own material, scatter the bundle and train -- bit-exact vs the oracle (which uses the
# dealer seed), without either party ever holding the dealer seed or the peer's shares.
# ---------------------------------------------------------------------------------------------
BUNDLE_TASK, BUNDLE_STEPS = "mlp", 2


def _party_bundled(rank, port, outdir, seed_p):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import synth
    from paper_conf_icpp_chenzzzz020_b200.parallel import make_dp, make_transport
    from paper_conf_icpp_chenzzzz020_b200.train import PartyTrainer
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=2)
    torch.cuda.set_device(0)
    xp = make_transport(rank, 1 - rank, kind="peer")
    dp = make_dp([rank], rank)
    dev = lambda name: torch.from_numpy(np.load(os.path.join(outdir, name))).cuda()  # noqa: E731
    Wi = synth.init_weights(BUNDLE_TASK)
    w_share = [dev(f"w{layer}_{rank}.npy") for layer in range(len(Wi))]
    tr = PartyTrainer(BUNDLE_TASK, Wi, rank, xp, dp=dp, w_share=w_share, dealer_seed=seed_p, deal_role=rank + 1)
    for s in range(BUNDLE_STEPS):
        bpath = os.path.join(outdir, f"bundle{s}_{rank}.npy")
        tr.model.deal_party(s, rank, dev(f"bundle{s}_{rank}.npy") if np.load(bpath).size else None)
        tr.model.party_train_step(rank, xp, dp, dev(f"x{s}_{rank}.npy"), dev(f"y{s}_{rank}.npy"), s)
        torch.cuda.synchronize()
        for layer in range(tr.model.n_layers):
            np.save(os.path.join(outdir, f"{BUNDLE_TASK}_s{s}_l{layer}_{rank}.npy"), tr.my_master_share(layer).cpu().numpy())
    tr.close()
    xp.close()
    dp.close()
    dist.destroy_process_group()


def test_split_training_with_dealer_bundles(tmp_path):
    import synth
    from paper_conf_icpp_chenzzzz020_b200 import build, psml
    from paper_conf_icpp_chenzzzz020_b200.train import DEALER_SEED, SecureTrainer
    build.build()
    torch.cuda.set_device(0)
    Wi = synth.init_weights(BUNDLE_TASK)
    dealer = SecureTrainer(BUNDLE_TASK, Wi)          # the client + dealer: holds the dealer seed
    for layer in range(dealer.model.n_layers):
        W = dealer.model.get_master(layer)
        for p in range(2):
            np.save(tmp_path / f"w{layer}_{p}.npy", W[p].cpu().numpy())
    sizes = []
    for s in range(BUNDLE_STEPS):
        X, Y = synth.batch(BUNDLE_TASK, s)
        Xs, Ys = dealer.share_batch(torch.from_numpy(X), torch.from_numpy(Y), s)
        for p in range(2):
            np.save(tmp_path / f"x{s}_{p}.npy", Xs[p].cpu().numpy())
            np.save(tmp_path / f"y{s}_{p}.npy", Ys[p].cpu().numpy())
            b = dealer.model.deal_bundle(s, p)
            sizes.append(b.numel())
            np.save(tmp_path / f"bundle{s}_{p}.npy", b.cpu().numpy())
    torch.cuda.synchronize()
    dealer.close()
    assert sizes[0] == 0 and sizes[1] > 0     # party 0 derives all of its A2B-mode material itself
    seeds = [psml.dealer_party_seed(DEALER_SEED, p) for p in range(2)]
    port = _free_port()
    ctx = mp.get_context("spawn")
    procs = [ctx.Process(target=_party_bundled, args=(p, port, str(tmp_path), seeds[p])) for p in range(2)]
    for pr in procs:
        pr.start()
    for pr in procs:
        pr.join(600)
        assert pr.exitcode == 0
    _check_against_oracle(tmp_path, [(BUNDLE_TASK, BUNDLE_STEPS)])
