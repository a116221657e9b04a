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
