#!/usr/bin/env python
"""Benchmark: secure MNIST-shaped MLP training samples/s (BASELINE.json metric, config 3) on
B200, plus the ring-GEMM TOPS figure of config 5, one JSON line on rank 0.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl reference]

A step = one pass of the whole hot path over one minibatch of 128 synthetic MNIST-shaped rows:
client encode + share of the batch (plaintext already in HBM), dealer material for the step
(triplets, MSB material), and the online secure step (masking, openings, Eq. 8 ring GEMMs,
truncation, secure ReLU / Eq. 9, backprop, master-weight update) -- DESIGN.md "Measurement".
N > 1 (torchrun): the split deployment -- party 0 on GPU k, party 1 on GPU k + N/2, N/2 pairs
each on its own 128 rows (weak scaling), every opening one peer-memory exchange over NVLink,
per-party NCCL all-reduce of the gradient shares, one CUDA graph per party step
(`--deployment coresident`: one co-resident pair per GPU instead; `--scaling strong`: ONE global
batch of 128 rows split over the pairs with the row-sliced dealer layout).
Timing: W untimed warm-up steps, then K steps each bracketed by CUDA events on the launching
stream with a 256 MiB L2 flush between steps (outside the events); barrier + synchronize around
the timed region; the max over ranks.  `--impl reference` times the CPU oracle instead.
"""
import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "secure training samples/s (MNIST MLP) at 1/2/4/8 B200; ring-GEMM TOPS vs INT8 peak"
WORKLOADS = {
    "mlp": "secure MLP 784-128-128-10 training with secure ReLU, batch 128, MNIST-shaped synthetic",
    "linreg": "secure linear regression training, MNIST-shaped synthetic 60000x784, batch 128",
    "logreg": "secure logistic regression training (Eq. 9 sigmoid), MNIST-shaped synthetic, batch 128",
    "cnn": "secure CNN (conv 5x5x16 as im2col ring GEMM, FC 64, FC 10) training, CIFAR-10-shaped "
           "synthetic 3x32x32, batch 128",
}
TASK, BATCH = "mlp", 128
WORKLOAD = WORKLOADS[TASK]
INT8_DENSE_PEAK_TOPS = 4500.0   # B200 nominal dense INT8 (B200_PROFILING / NVIDIA spec), context


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=1000)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-ring-gemm", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--mask-reuse", action="store_true",
                    help="split deployment: SecureML forward/backward mask reuse (DESIGN.md R26)")
    ap.add_argument("--compare", default="a2b", choices=["a2b", "fss"],
                    help="secure comparison of ReLU / Eq. 9: A2B chain (R9) or one-round FSS (R22)")
    ap.add_argument("--no-secondary", action="store_true", help="skip the other configs' figures")
    ap.add_argument("--no-classes", action="store_true",
                    help="skip the CUPTI kernel-class leg (required under ncu: one CUPTI client at a time)")
    ap.add_argument("--task", default="mlp", choices=sorted(WORKLOADS),
                    help="headline is mlp (BASELINE metric); others are secondary configs")
    ap.add_argument("--sweep", default=None, metavar="N1,N2,...",
                    help="config-5 ring GEMM sweep (e.g. 512,1024,2048,4096,8192); prints JSON lines")
    ap.add_argument("--deployment", default="auto", choices=["auto", "coresident", "split"],
                    help="split: party 0 and party 1 on different GPUs (ranks k and k + N/2), every "
                         "opening round one peer-memory exchange over NVLink (SURVEY 8(e)); "
                         "coresident: both parties of a pair on one GPU; auto (default): split for "
                         "N >= 2, coresident for N = 1")
    ap.add_argument("--scaling", default="weak", choices=["weak", "strong"],
                    help="N > 1: weak = 128 rows per pair (global batch 128 x pairs); strong = ONE global "
                         "batch of 128 rows split over the pairs with the row-sliced dealer layout "
                         "(SURVEY C16, DESIGN.md R28)")
    a = ap.parse_args()
    global TASK, WORKLOAD
    TASK, WORKLOAD = a.task, WORKLOADS[a.task]
    return a


# ---------------------------------------------------------------------------------------------
# clocks sampler (nvidia-smi during the timed region)
# ---------------------------------------------------------------------------------------------
REASON_BITS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
               0x8: "hw_slowdown", 0x10: "sync_boost", 0x20: "sw_thermal_slowdown",
               0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown",
               0x100: "display_clock_setting"}


class ClockSampler:
    def __init__(self, index):
        self.index = index
        self.samples = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), "--query-gpu=clocks.sm,clocks.max.sm,"
                 "clocks_event_reasons.active", "--format=csv,noheader,nounits", "-lms", "20"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.thread = threading.Thread(target=self._read, daemon=True)
            self.thread.start()
            # nvidia-smi takes a while to start: wait for its first sample so the sampling is live
            # when the timed region begins, then keep only samples taken inside the region
            t0 = time.time()
            while not self.samples and time.time() - t0 < 15.0 and self.proc.poll() is None:
                time.sleep(0.01)
            self.samples.clear()
        except OSError:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            parts = [p.strip() for p in line.split(",")]
            if len(parts) >= 3:
                try:
                    self.samples.append((float(parts[0]), float(parts[1]), int(parts[2], 16)))
                except ValueError:
                    pass

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except subprocess.TimeoutExpired:
                self.proc.kill()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}
        load = [s for s in self.samples if not (s[2] & 0x1)] or self.samples
        reasons = set()
        for s in load:
            for bit, name in REASON_BITS.items():
                if s[2] & bit:
                    reasons.add(name)
        return {"sm_mhz": statistics.median(s[0] for s in load),
                "sm_max_mhz": max(s[1] for s in load), "reasons": sorted(reasons),
                "samples": len(load)}


# ---------------------------------------------------------------------------------------------
# our arm
# ---------------------------------------------------------------------------------------------
def dist_setup(args):
    import torch
    import torch.distributed as dist
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # PSML_DIST_BACKEND=gloo + PSML_SHARE_GPU=1: all ranks on cuda:0 over gloo -- exercises the
    # data-parallel path on a one-GPU box (not a performance configuration).
    backend = os.environ.get("PSML_DIST_BACKEND", "nccl")
    if os.environ.get("PSML_SHARE_GPU") == "1":
        local = 0
    if world > 1:
        torch.cuda.set_device(local)
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    else:
        torch.cuda.set_device(0)
    return world, rank, local


def pair_batch(args, s, pair, pairs, u8=False):
    """Minibatch rows of pair `pair` of `pairs` for step s: its own 128 rows (weak scaling) or its
    slice of ONE global batch of 128 rows (strong scaling, parallel.strong_rows)."""
    import synth
    gen = synth.batch_u8 if u8 else synth.batch
    if args.scaling == "strong" and pairs > 1:
        from paper_conf_icpp_chenzzzz020_b200.parallel import strong_rows
        X, Y = gen(TASK, s, BATCH)
        r = strong_rows(pair, pairs, BATCH)
        return X[r], Y[r]
    return gen(TASK, s, BATCH, pair=pair, n_pairs=pairs)


def per_pair_rows(args, pairs):
    return BATCH // pairs if (args.scaling == "strong" and pairs > 1) else BATCH


def max_over_ranks(x, world):
    if world == 1:
        return x
    import torch
    import torch.distributed as dist
    t = torch.tensor([x], dtype=torch.float64, device="cuda")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def bench_ours(args):
    import numpy as np
    import torch
    import torch.distributed as dist

    import synth
    from paper_conf_icpp_chenzzzz020_b200 import build, psml
    from paper_conf_icpp_chenzzzz020_b200.parallel import ring_allreduce_
    from paper_conf_icpp_chenzzzz020_b200.train import SecureTrainer

    build.build()
    world, rank, local = dist_setup(args)
    dev = torch.device("cuda", local)
    K, W = args.steps, args.warmup
    whole = ClockSampler(local).__enter__()   # clocks over the whole GPU-active bench
    strong = args.scaling == "strong" and world > 1
    rows = per_pair_rows(args, world)
    tr = SecureTrainer(TASK, synth.init_weights(TASK), batch=rows, pair_id=rank, strong_pairs=world if strong else 0)
    # plaintext minibatches resident in HBM (and pinned host copies for the e2e leg)
    nb = K + W
    Xs, Ys = [], []
    for s in range(nb):
        X, Y = pair_batch(args, s, rank, world)
        Xs.append(torch.from_numpy(np.ascontiguousarray(X)).to(dev))
        Ys.append(torch.from_numpy(np.ascontiguousarray(Y)).to(dev))
    # e2e leg: the client's own form of the same batches -- 8-bit pixels and (one-hot tasks)
    # class indices -- in pinned host memory; they share bit-identically to the float64 batches
    Xh, Yh = [], []
    for s in range(nb):
        q, y = pair_batch(args, s, rank, world, u8=True)
        q = np.ascontiguousarray(q)
        Xh.append(torch.from_numpy(q).pin_memory())
        Yh.append(torch.from_numpy(np.ascontiguousarray(y)).pin_memory())
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream()

    def graph_step(s, X, Y):
        # client encode + share into the captured buffers, then one graph replay (dealer +
        # online step [+ update]); data parallel: NCCL all-reduce of gradient shares + update
        tr.graph_step(X, Y, s)
        if world > 1:
            ring_allreduce_(tr.grad_tensor())
            tr.model.apply_update(extra_shift=tr.update_shift(world))

    def one_step(s, X, Y, online_only=False, shares=None):
        if online_only:
            tr.model.train_step(*shares, s) if world == 1 else tr.step_dp(*shares, s, deal=False)
            return
        Xsh, Ysh = tr.share_batch(X, Y, s)
        if world == 1:
            tr.step_shares(Xsh, Ysh, s)
        else:
            tr.step_dp(Xsh, Ysh, s)

    def timed(fn, n_steps, base):
        evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
               for _ in range(n_steps)]
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        for i in range(n_steps):
            flush.zero_()
            evs[i][0].record(stream)
            fn(base + i)
            evs[i][1].record(stream)
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        return sum(a.elapsed_time(b) for a, b in evs) / 1e3

    for s in range(W):
        one_step(s, Xs[s], Ys[s])
    torch.cuda.synchronize()
    EB = 10 ** 6   # eager comparison steps use their own step ids (fresh dealer material)
    t_eager = max_over_ranks(timed(lambda s: one_step(s, Xs[(s - EB) % nb], Ys[(s - EB) % nb]), K, EB),
                             world)
    tr.capture(with_update=(world == 1))
    graph_step(W - 1, Xs[0], Ys[0])    # warm the graph once (primes the dealer pipeline for step W)
    torch.cuda.synchronize()
    l0 = psml.kernel_launch_count()
    n_nodes = tr.graph_kernel_nodes()
    with ClockSampler(local) as clk:
        t_dev = timed(lambda s: graph_step(s, Xs[s], Ys[s]), K, W)
    launches = psml.kernel_launch_count() - l0
    t_dev = max_over_ranks(t_dev, world)

    # online-only CUDA graph (diagnostic): re-capture the step without the dealer branch and
    # replay it on material dealt once (timing only -- a real run never reuses triplets)
    t_on_graph = None
    if world == 1:
        tr.model.deal(0)
        gs = torch.cuda.Stream()
        gs.wait_stream(stream)
        with torch.cuda.stream(gs):
            tr.model.capture_step(tr.Xbuf, tr.Ybuf, with_deal=False, with_update=True, pipelined=False,
                                  stream=gs, unsafe_reuse_material=True)
        stream.wait_stream(gs)
        tr.model.step_graph(0)
        torch.cuda.synchronize()
        t_on_graph = timed(lambda s: tr.model.step_graph(0), K, 0)
        tr.capture(with_update=True)   # restore the pipelined graph for the e2e leg
        tr._next_dealt = None

    # online-only (dealer material generated before each step, outside the events)
    evs = []
    for i in range(K):
        s = W + K + i
        Xsh, Ysh = tr.share_batch(Xs[i % nb], Ys[i % nb], s)
        tr.deal(s)
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        one_step(s, None, None, online_only=True, shares=(Xsh, Ysh))
        b.record(stream)
        evs.append((a, b))
    torch.cuda.synchronize()
    t_on = max_over_ranks(sum(a.elapsed_time(b) for a, b in evs) / 1e3, world)

    # e2e through the public API with host buffers: H2D plaintext batch, full step, D2H yhat
    h2d = Xh[0].numel() * Xh[0].element_size() + Yh[0].numel() * Yh[0].element_size()
    out_host = torch.empty((2, rows, Ys[0].shape[1]), dtype=torch.uint64).pin_memory()
    d2h = out_host.numel() * 8

    def e2e_step(s):
        i = (s - 2 * (W + K)) % nb
        if world == 1:
            # one library call: H2D pixels + labels, client encode/share, the captured step, D2H
            # of both parties' prediction shares (psml_model_step_host)
            tr.graph_step_host(Xh[i], Yh[i], s, out_host)
            return
        X = Xh[i].to(dev, non_blocking=True)
        Y = Yh[i].to(dev, non_blocking=True)
        graph_step(s, X, Y)
        # the step's result: both parties' prediction shares of this batch
        y0, y1 = tr.last_yhat()
        out_host[0].view(-1).copy_(y0, non_blocking=True)
        out_host[1].view(-1).copy_(y1, non_blocking=True)
    t_e2e = max_over_ranks(timed(e2e_step, K, 2 * (W + K)), world)

    # secure inference (the forward half): client share + inference dealer + forward
    def infer_step(s):
        i = s % nb
        Xsh, _ = tr.share_batch(Xs[i], Ys[i], s)
        tr.infer_shares(Xsh, s)
    t_inf = max_over_ranks(timed(infer_step, K, 10 * (W + K)), world)

    samples = rows * K * world
    result = {
        "metric": METRIC, "value": samples / t_dev, "unit": "samples/s", "n_gpus": world,
        "steps": K, "warmup": W, "ms_per_step": 1e3 * t_dev / K, "higher_is_better": True,
        "scaling": "strong" if strong else "weak", "vs_baseline": None, "dtype": "u64",
        "data": ("synthetic (CIFAR-shaped 3x32x32 8-bit pixels; teacher-CNN labels)" if TASK == "cnn" else
                 "synthetic (MNIST-shaped 8-bit pixels, 81% zeros; teacher labels)"),
        "config": arm_config(world, args.scaling),
        "online_samples_per_s": samples / t_on,
        "online_graph_samples_per_s": (samples / t_on_graph) if t_on_graph else None,
        "eager_samples_per_s": samples / t_eager,
        "infer_samples_per_s": samples / t_inf,
        "cuda_graph": {"kernel_nodes_per_step": n_nodes,
                       "note": "value/e2e replay one captured graph per step (dealer + online "
                               "step + update); online/eager figures use per-kernel launches"},
        "e2e": {"value": samples / t_e2e, "unit": "samples/s", "h2d_bytes_per_step": h2d,
                "d2h_bytes_per_step": d2h},
        "gpu_launches": int(launches),
        "clocks": clk.summary(),
    }
    # Per-kernel-class device time of the headline step, from CUPTI kernel records (torch.profiler)
    # of K replays of the same pipelined graph; algorithmic work per launch from the library's
    # counters over K eager steps (psml_prof: ring MACs for GEMM classes, bytes otherwise).
    work = {}
    base = 3 * (W + K)
    for cls in (psml.PROF_GEMM, psml.PROF_TC, psml.PROF_MSB, psml.PROF_HAD, psml.PROF_DEALER, psml.PROF_MASK):
        psml.prof_enable(cls)
        psml.prof_read()
        for i in range(K):
            one_step(base + i, Xs[i % nb], Ys[i % nb])
        _, n, w = psml.prof_read()
        psml.prof_enable(-1)
        base += K
        work[PROF_CLASS[cls]] = (n / K, w / max(n, 1))
    classes = None
    if not args.no_classes and t_on_graph:
        tr.model.deal(0)
        gs = torch.cuda.Stream()
        gs.wait_stream(stream)
        with torch.cuda.stream(gs):
            tr.model.capture_step(tr.Xbuf, tr.Ybuf, with_deal=False, with_update=True, pipelined=False,
                                  stream=gs, unsafe_reuse_material=True)
        stream.wait_stream(gs)
        classes = cupti_classes(lambda i: tr.model.step_graph(0), lambda i: tr.model.deal(base + i), K,
                                1e3 * t_on_graph / K, work)
    mac_peak = mac_peak_tmacs()
    int8 = int8_peak_tops()
    if classes:
        result["kernel_classes"] = classes
        result["roofline"] = roofline(classes, mac_peak, int8)
        result["offline"] = offline_figure(classes["dealer"], samples / K)
    gemm_macs = sum(w[0] * w[1] for c, w in work.items() if c in ("ring_gemm_cuda_core", "ring_gemm_tcgen05"))
    step_ops = 36 * 2 * gemm_macs
    result["step_int8_fraction"] = {
        "useful_limb_ops_per_step": step_ops,
        "achieved_tops": step_ops / (result["ms_per_step"] / 1e3) / 1e12, "peak_tops": int8[0],
        "frac": step_ops / (result["ms_per_step"] / 1e3) / 1e12 / int8[0], "peak_source": int8[1],
        "note": "every Beaver product of the step (both parties, K' = 2K) counted as 36 useful "
                "limb-pair MMAs x 2 ops per ring MAC, whichever unit ran it"}
    whole.__exit__()
    result["clocks_timed_region"] = result["clocks"]
    result["clocks"] = whole.summary()
    result["clocks"]["window"] = "whole bench (warm-up, timed legs, profiling legs)"
    return result, tr, world, rank


def bench_split(args):
    """Split deployment (the north_star multi-GPU layout): N/2 party pairs, pair k =
    (rank k: party 0, rank k + N/2: party 1), each pair on its own 128 rows (weak scaling).  Every
    opening round is one exchange kernel over the pair's peer-memory mailboxes (CUDA IPC, NVLink
    stores between the two GPUs); each party sums its untruncated gradient share over its N/2
    GPUs with the library-owned NCCL all-reduce; the whole party step (dealer of the next step on
    a forked branch, online phase with its exchanges, all-reduce, update) is one CUDA graph."""
    import numpy as np
    import torch
    import torch.distributed as dist

    import synth
    from paper_conf_icpp_chenzzzz020_b200 import build, psml
    from paper_conf_icpp_chenzzzz020_b200.parallel import make_dp, make_transport, pair_layout
    from paper_conf_icpp_chenzzzz020_b200.train import PartyTrainer

    build.build()
    world, rank, local = dist_setup(args)
    party, pair, peer = pair_layout(world)(rank)
    half = world // 2
    groups = [dist.new_group(list(range(q * half, (q + 1) * half))) for q in range(2)]
    dev = torch.device("cuda", local)
    K, W = args.steps, args.warmup
    cap = (96 << 20) if TASK == "cnn" else (8 << 20)
    xp = make_transport(party, peer, kind=os.environ.get("PSML_XPORT", "peer"), capacity_bytes=cap)
    dp = make_dp(list(range(party * half, (party + 1) * half)), rank, groups[party])
    strong = args.scaling == "strong" and half > 1
    rows = per_pair_rows(args, half)
    tr = PartyTrainer(TASK, synth.init_weights(TASK), party, xp, batch=rows, pair_id=pair, dp=dp,
                      mask_reuse=args.mask_reuse, compare=args.compare, strong_pairs=half if strong else 0)
    nb = min(K + W, 64)
    Xs, Ys, Xh, Yh = [], [], [], []
    for s in range(nb):
        X, Y = pair_batch(args, s, pair, half)
        Xs.append(torch.from_numpy(np.ascontiguousarray(X)).to(dev))
        Ys.append(torch.from_numpy(np.ascontiguousarray(Y)).to(dev))
        q, y = pair_batch(args, s, pair, half, u8=True)
        Xh.append(torch.from_numpy(np.ascontiguousarray(q)).pin_memory())
        Yh.append(torch.from_numpy(np.ascontiguousarray(y)).pin_memory())
    stream = torch.cuda.current_stream()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)

    def timed(fn, n, base):
        evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(n)]
        dist.barrier()
        torch.cuda.synchronize()
        for i in range(n):
            flush.zero_()
            evs[i][0].record(stream)
            fn(base + i)
            evs[i][1].record(stream)
        torch.cuda.synchronize()
        dist.barrier()
        return max_over_ranks(sum(a.elapsed_time(b) for a, b in evs) / 1e3, world)

    # eager warm-up, then capture the party step (the capture issues every exchange once)
    for s in range(W):
        X_i, Y_i = tr.share_batch(Xs[s % nb], Ys[s % nb], s)
        tr.step_party(X_i, Y_i, s)
    torch.cuda.synchronize()
    b0, x0 = xp.stats()
    tr.capture_party(pipelined=True)
    b1, x1 = xp.stats()

    def step(s):
        X_i, Y_i = tr.share_batch(Xs[s % nb], Ys[s % nb], s)
        tr.graph_step_party(X_i, Y_i, s)

    step(W)
    torch.cuda.synchronize()
    l0 = psml.kernel_launch_count()
    with ClockSampler(local) as clk:
        t_dev = timed(step, K, W + 1)
    launches = psml.kernel_launch_count() - l0
    out_host = torch.empty(rows * Ys[0].shape[1], dtype=torch.uint64).pin_memory()
    from paper_conf_icpp_chenzzzz020_b200.train import _wrap_device_ptr

    def e2e(s):
        i = s % nb
        X_i, Y_i = tr.share_batch(Xh[i], Yh[i], s)     # H2D of pixels + class indices, client share
        tr.graph_step_party(X_i, Y_i, s)
        ptrs = tr.model.output()
        out_host.copy_(_wrap_device_ptr(ptrs[party], ptrs[2], "<u8"), non_blocking=True)
    t_e2e = timed(e2e, K, W + K + 1)
    samples = rows * K * half
    return {
        "metric": METRIC, "value": samples / t_dev, "unit": "samples/s", "n_gpus": world,
        "steps": K, "warmup": W, "ms_per_step": 1e3 * t_dev / K, "higher_is_better": True,
        "scaling": "strong" if strong else "weak", "vs_baseline": None, "dtype": "u64",
        "data": "synthetic (MNIST-shaped 8-bit pixels, 81% zeros; teacher labels)",
        "config": {"workload": WORKLOAD, "deployment": "split (party 0 on GPU k, party 1 on GPU k + N/2)",
                   "global_batch": rows * half, "per_pair_batch": rows, "pairs": half,
                   "ring": "Z_2^64, 13 fractional bits", "parallelism": f"{half} pairs x 2 parties",
                   "transport": xp_kind(), "mask_reuse": bool(args.mask_reuse), "compare": args.compare,
                   "l2": "256 MiB flush between timed steps (outside the events)",
                   "step": "client share, dealer of the next step (forked graph branch), online step "
                           "with one exchange per opening round, per-party gradient all-reduce, update: "
                           "one CUDA graph per party"},
        "exchanges_per_step": x1 - x0, "bytes_sent_per_step_per_party": b1 - b0,
        "e2e": {"value": samples / t_e2e, "unit": "samples/s",
                "h2d_bytes_per_step": Xh[0].numel() + Yh[0].numel(),
                "d2h_bytes_per_step": out_host.numel() * 8},
        "gpu_launches": int(launches), "clocks": clk.summary(),
        "roofline": None,
    }, rank


def xp_kind():
    return {"peer": "peer-memory mailboxes (CUDA IPC, NVLink stores), one kernel per exchange",
            "nccl": "NCCL send/recv", "callback": "host-staged"}[os.environ.get("PSML_XPORT", "peer")]


def measured_peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except (OSError, ValueError):
        return {}


def committed_traffic(name):
    """DRAM bytes per launch of kernel class `name` from the newest committed ncu --set full
    capture that has it (profiles/r0*_traffic.json, written by tools/traffic.py), or None."""
    import glob
    for f in sorted(glob.glob(os.path.join(ROOT, "profiles", "r0*_traffic.json")), reverse=True):
        try:
            t = json.load(open(f))
            # the committed summary this value is read from (its source capture stays out of the tree)
            return t[name]["bytes_per_launch_avg"], f"{os.path.relpath(f, ROOT)} (from {t['source']})"
        except (OSError, ValueError, KeyError):
            continue
    return None, None


PROF_CLASS = {0: "ring_gemm_cuda_core", 1: "ring_gemm_tcgen05", 2: "msb_relu_eq9_rounds", 3: "hadamard_rounds",
              4: "dealer", 5: "beaver_mask"}
# kernel name -> class (CUPTI records); the dealer's Z = U V products are dealer work
KERNEL_CLASS = (("ring_gemm_cl_grouped", "dealer"), ("deal_prg", "dealer"), ("dealer_", "dealer"),
                ("hadamard_triplet", "dealer"), ("msb_dealer", "dealer"), ("prg_kernel", "dealer"),
                ("tc_seg", "ring_gemm_tcgen05"), ("tc_ring", "ring_gemm_tcgen05"),
                ("seg_gemm", "ring_gemm_cuda_core"), ("ring_gemm", "ring_gemm_cuda_core"),
                ("msb_", "msb_relu_eq9_rounds"), ("had_", "hadamard_rounds"), ("hadamard", "hadamard_rounds"),
                ("eq9", "hadamard_rounds"), ("open", "beaver_mask"), ("mask", "beaver_mask"),
                ("update", "update"), ("encode_share", "client_share"), ("client_share", "client_share"))


def kernel_class(name):
    for pat, cls in KERNEL_CLASS:
        if pat in name:
            return cls
    return "other"


def _kernel_records(fn, n):
    """CUPTI kernel records (name, start_ns, end_ns) of n calls of fn(i) (torch.profiler)."""
    import torch
    from torch.profiler import ProfilerActivity, profile
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        for i in range(n):
            fn(i)
        torch.cuda.synchronize()
    recs = []
    for e in prof.profiler.kineto_results.events():
        if "cuda" not in str(e.device_type()).lower():
            continue
        name = e.name()
        if name.startswith(("Memcpy", "Memset")) or "elementwise" in name or "Fill" in name:
            continue
        t0 = e.start_ns()
        recs.append((name, t0, t0 + e.duration_ns()))
    return recs


def attribute(recs):
    """Device time per kernel record with overlaps resolved in favour of the EARLIEST-started
    active kernel: under programmatic dependent launch a kernel's CTAs start while its
    predecessor still runs and wait (griddepcontrol.wait) -- that wait is the predecessor's time.
    The attributed times of a run sum to its busy wall time."""
    ev = sorted(recs, key=lambda r: r[1])
    out = [0.0] * len(ev)
    cover = None   # end of the time already attributed
    for i, (_, t0, t1) in enumerate(ev):
        lo = t0 if cover is None else max(t0, cover)
        if t1 > lo:
            out[i] = (t1 - lo) / 1e6   # ms
            cover = t1 if cover is None else max(cover, t1)
    return [(ev[i][0], out[i]) for i in range(len(ev))]


def cupti_classes(step_fn, deal_fn, K, ms_step_online, work):
    """Per-kernel-class device time: CUPTI kernel records of K replays of the online-phase graph
    (step_fn) and K dealer calls (deal_fn), each kernel's time attributed by `attribute`;
    work_per_launch from the library counters (`work`)."""
    import torch
    step_fn(-1)
    torch.cuda.synchronize()
    tot, cnt = {}, {}
    for fn in (step_fn, deal_fn):
        for name, ms in attribute(_kernel_records(fn, K)):
            c = kernel_class(name)
            if fn is deal_fn and c != "dealer":
                c = "dealer"
            tot[c] = tot.get(c, 0.0) + ms
            cnt[c] = cnt.get(c, 0) + 1
    out = {}
    for c in tot:
        n_step, w = work.get(c, (cnt[c] / K, 0.0))
        out[c] = {"ms_per_step": tot[c] / K, "share_of_online_step": tot[c] / K / ms_step_online,
                  "launches_per_step": cnt[c] / K, "ms_per_launch": tot[c] / cnt[c],
                  "work_per_launch": w, "work_launches_per_step_eager": n_step,
                  "source": "CUPTI kernel records (torch.profiler), overlap attributed to the earliest-started "
                            "kernel (PDL waits belong to the predecessor)"}
    online = sum(v["ms_per_step"] for k, v in out.items() if k != "dealer")
    out["_check"] = {"online_class_sum_ms": online, "online_graph_ms_per_step": ms_step_online,
                     "note": "online classes from the online-phase graph (dealer material replayed); "
                             "dealer from psml_model_deal calls"}
    return out


def mac_peak_tmacs():
    """Measured CUDA-core ring-MAC throughput (psml_bench_mac_peak, Z_2^64), T ring-MAC/s."""
    from paper_conf_icpp_chenzzzz020_b200 import psml
    try:
        return psml.bench_mac_peak(64) / 1e12, "measured: psml_bench_mac_peak (register-only u64 MAC chains, all SMs)"
    except Exception as e:   # noqa: BLE001
        return 148 * 64 / 3 * 1.965e9 / 1e12, f"derived (microbenchmark failed: {e})"


def roofline(classes, mac_peak, int8):
    """Roofline of the dominant kernel: the largest ONLINE-phase class of the step by CUPTI device
    time (the dealer runs concurrently with the online phase in the pipelined graph)."""
    online = [k for k in classes if k not in ("dealer", "client_share", "_check", "other", "update")]
    online = [k for k in online if k in PROF_CLASS.values()]
    name = max(online, key=lambda k: classes[k]["ms_per_step"])
    c = classes[name]
    sec = c["ms_per_launch"] / 1e3
    mp = measured_peaks()
    sel = "largest online-phase kernel class by CUPTI device time (dealer overlapped)"
    if name == "ring_gemm_tcgen05":
        ach = 36 * 2 * c["work_per_launch"] / sec / 1e12
        r = {"bound": "tensor", "class": name, "kernel": "tc_seg_kernel (tcgen05 kind::i8, in-kernel limb split)",
             "achieved": ach, "peak": int8[0], "unit": "TOPS", "frac": ach / int8[0], "peak_source": int8[1]}
    elif name == "ring_gemm_cuda_core":
        ach = c["work_per_launch"] / sec / 1e12
        r = {"bound": "alu", "class": name, "kernel": "seg_gemm_kernel (CUDA-core two-segment Beaver GEMM)",
             "achieved": ach, "peak": mac_peak[0], "unit": "T ring-MAC/s", "frac": ach / mac_peak[0],
             "peak_source": mac_peak[1]}
    else:
        peak = mp.get("hbm_gbs", 6650.0)
        ach = c["work_per_launch"] / sec / 1e9
        r = {"bound": "hbm", "class": name, "kernel": name, "achieved": ach, "peak": peak, "unit": "GB/s",
             "frac": ach / peak, "peak_source": "measured" if "hbm_gbs" in mp else "fallback"}
    r["selection"] = sel
    r["traffic"], src = committed_traffic(name)
    if src:
        r["traffic_unit"], r["traffic_source"] = "bytes per launch", src
    return r


def offline_figure(dealer, samples_per_step):
    """Offline phase (Table 3): the dealer's material for one step --
    ChaCha20 streams (U/V/Z_0 masks, AND triplets, daBits, Hadamard triplets) plus the grouped
    Z_1 = U V - Z_0 products -- timed alone (class 'dealer').  The PRG is bound by the ALU pipe:
    a ChaCha20 block is 80 quarter rounds x (4 LOP3 + 4 SHF) = 640 ALU-pipe ops (the 4 adds per
    quarter round issue as IMAD on the FMA pipe, cuobjdump of deal_prg_kernel); ALU-pipe peak =
    148 SMs x 64 lanes/clk x 1965 MHz (B300_MICROARCH: alu rt_SMSP = 2).  The class time includes
    the Z = U V products, so the fraction is a lower bound for the PRG kernel."""
    sec = dealer["ms_per_step"] / 1e3
    blocks = dealer["work_per_launch"] * dealer.get("work_launches_per_step_eager", dealer["launches_per_step"])
    peak_blocks = 148 * 64 * 1.965e9 / 640
    return {"ms_per_step": dealer["ms_per_step"], "samples_per_s": samples_per_step / sec,
            "chacha20_blocks_per_step": blocks, "prg_output_GBps": blocks * 64 / sec / 1e9,
            "prg_alu_roofline": {"bound": "alu", "achieved": blocks / sec / 1e9, "peak": peak_blocks / 1e9,
                                 "unit": "G ChaCha20 blocks/s", "frac_lower_bound": blocks / sec / peak_blocks}}


_INT8 = None


def int8_peak_tops():
    """Dense INT8 tensor ceiling MEASURED on this GPU: cuBLASLt IMMA via torch._int_mm on 8192^3
    int8 operands (2 n^3 ops, best of 5, CUDA events); fallback: measured bf16 burst x 2."""
    global _INT8
    if _INT8 is not None:
        return _INT8
    import torch
    try:
        n = 8192
        a = torch.randint(-128, 127, (n, n), dtype=torch.int8, device="cuda")
        b = torch.randint(-128, 127, (n, n), dtype=torch.int8, device="cuda").t().contiguous().t()
        for _ in range(2):
            torch._int_mm(a, b)
        best = 1e30
        for _ in range(5):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            torch._int_mm(a, b)
            e1.record()
            torch.cuda.synchronize()
            best = min(best, e0.elapsed_time(e1))
        _INT8 = (2.0 * n ** 3 / (best / 1e3) / 1e12, "measured: torch._int_mm (cuBLASLt INT8) 8192^3, best of 5")
        del a, b
    except Exception as e:   # noqa: BLE001
        mp = measured_peaks()
        bf = mp.get("bf16_tflops", 1590.0)
        _INT8 = (2.0 * bf, f"measured bf16 burst x nominal int8/bf16 ratio 2 (torch._int_mm failed: {e})")
    return _INT8


def ring_gemm_figure(n=4096, l=64, reps=5):
    """BASELINE config 5 kernel: plain C = A B mod 2^l, n^3, timed with CUDA events."""
    import torch
    from paper_conf_icpp_chenzzzz020_b200 import psml
    ctx = psml.Ctx(l=l)
    ring = ctx.ring
    A = psml.prg_fill(ring, 1, psml.tag("bA"), 0, n * n).view(n, n)
    B = psml.prg_fill(ring, 1, psml.tag("bB"), 0, n * n).view(n, n)
    C = psml.empty(0, l, (n, n))
    psml.ring_gemm(ctx, A, B, out=C)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    tot = 0.0
    for _ in range(reps):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda._sleep(200_000)   # device busy while the host submits: events bracket device time
        a.record()
        psml.ring_gemm(ctx, A, B, out=C)
        b.record()
        torch.cuda.synchronize()
        tot += a.elapsed_time(b)
    ms = tot / reps
    pairs = 36 if l == 64 else 10
    useful = pairs * 2.0 * n ** 3
    ctx.close()
    traffic, tsrc = None, None
    if n == 4096:
        g, tsrc = committed_traffic("ring_gemm_tc_l64" if l == 64 else "ring_gemm_tc_l32")
        sp, _ = committed_traffic("ring_gemm_limb_split")
        traffic = (g + sp) if (g and sp) else None
    tops = useful / (ms / 1e3) / 1e12
    peak, src = int8_peak_tops()
    return {"n": n, "l": l, "ms": ms, "useful_limb_tops": tops,
            "frac_of_int8_dense_spec_4500": tops / INT8_DENSE_PEAK_TOPS,
            "roofline": {"bound": "tensor",
                         "kernel": ("tc_seg_kernel (tcgen05 kind::i8, in-kernel limb split, one launch)" if n <= 1024
                                    else "tc_ring_gemm (tcgen05 kind::i8 limb planes)"),
                         "achieved": tops, "peak": peak, "unit": "TOPS", "frac": tops / peak,
                         "traffic": traffic, "traffic_unit": "bytes per call (limb split + GEMM)",
                         "traffic_source": tsrc, "algorithmic_bytes": 2 * n * n * (l // 8) + n * n * (l // 8),
                         "peak_source": src},
            "ring_tmacs": n ** 3 / (ms / 1e3) / 1e12}


def beaver_latency_figure(reps=2000):
    """BASELINE config 1: one Beaver secure matmul A 128x784 . B 784x1 in Z_2^64 (both parties
    co-resident, one linear-regression minibatch), per-call device latency p50/p99 over `reps`
    calls (CUDA events around each call), beside the oracle's per-call time on the same inputs."""
    import numpy as np
    import torch
    from paper_conf_icpp_chenzzzz020_b200 import psml
    M, K, N = 128, 784, 1
    ctx = psml.Ctx(l=64)
    ring = ctx.ring
    A = psml.share(ring, 7, 1, psml.prg_fill(ring, 1, psml.tag("cA"), 0, M * K).view(M, K))
    B = psml.share(ring, 7, 2, psml.prg_fill(ring, 1, psml.tag("cB"), 0, K * N).view(K, N))
    U, V, Z = psml.triplet_gen(ctx, 3, 0, M, K, N)
    C = psml.empty_pair((M, N), 64)
    for _ in range(20):
        psml.secure_matmul(ctx, A, B, U, V, Z, M, K, N, trunc=13, out=C)
    l0 = psml.kernel_launch_count()
    psml.secure_matmul(ctx, A, B, U, V, Z, M, K, N, trunc=13, out=C)
    per_call = psml.kernel_launch_count() - l0
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
    torch.cuda.synchronize()
    # Device latency per call: each chunk of calls is enqueued behind a GPU sleep long enough for
    # the host to submit the whole chunk, so the calls run back to back and the events bracket
    # device time only (not the host's ctypes/launch overhead).
    chunk = 100
    for c0 in range(0, reps, chunk):
        torch.cuda._sleep(20_000_000)
        for a, b in evs[c0:c0 + chunk]:
            a.record()
            psml.secure_matmul(ctx, A, B, U, V, Z, M, K, N, trunc=13, out=C)
            b.record()
        torch.cuda.synchronize()
    us = np.array([a.elapsed_time(b) * 1e3 for a, b in evs])
    # the oracle on the same shares and triplet
    from oracle import core as orc
    host = lambda t: t.cpu().numpy()  # noqa: E731
    An, Bn = [host(t) for t in A], [host(t) for t in B]
    trip = [host(t) for t in (U[0], U[1], V[0], V[1], Z[0], Z[1])]
    t0 = time.perf_counter()
    n_or = 0
    while time.perf_counter() - t0 < 1.0:
        want = orc.beaver_matmul(An, Bn, trip, trunc=13)
        n_or += 1
    t_or = (time.perf_counter() - t0) / n_or * 1e6
    ok = all(np.array_equal(host(C[i]), want[i]) for i in range(2))
    ctx.close()
    return {"config": "single Beaver secure matmul, 2 parties co-resident, Z_2^64, A 128x784 . B 784x1",
            "p50_us": float(np.percentile(us, 50)), "p99_us": float(np.percentile(us, 99)),
            "reps": reps, "launches_per_call": int(per_call), "bitexact_vs_oracle": bool(ok),
            "oracle_us_per_call": t_or, "oracle_cores": orc.num_threads()}


def tev(fn, reps):
    import torch
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    fn()
    ts = []
    for _ in range(reps):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda._sleep(200_000)   # ~0.1 ms of GPU work: the host submits fn() meanwhile, so the
        a.record()                   # events bracket device time, not host launch latency
        fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return sorted(ts)[len(ts) // 2]


def cfg5_sweep(ns):
    """BASELINE config 5 sweep (bench.py --sweep): plain ring GEMM n^3 for l = 64 / 32 on tcgen05 (CUDA
    cores to 2048), the co-resident Beaver secure matmul at every n, and -- the cpu_baseline leg --
    the CPU oracle's ring matmul (all host threads) at n <= 2048 with bit-exact parity of the GPU
    result, n^3-extrapolated above (labelled).  One JSON line per (n, l)."""
    import numpy as np
    import torch
    from oracle import core as orc
    from paper_conf_icpp_chenzzzz020_b200 import psml
    oracle_t = {}
    for n in ns:
        for l in (64, 32):
            pairs = 36 if l == 64 else 10
            ring = psml.Ring(l, 13)
            A = psml.prg_fill(ring, 1, psml.tag("bA"), 0, n * n).view(n, n)
            B = psml.prg_fill(ring, 1, psml.tag("bB"), 0, n * n).view(n, n)
            C = psml.empty(0, l, (n, n))
            reps = 5 if n >= 4096 else 10
            row = {"n": n, "l": l}
            for be, name in ((2, "tcgen05"), (1, "cuda_core")):
                if be == 1 and n > 2048:
                    continue
                ctx = psml.Ctx(l=l, backend=be)
                ms = tev(lambda: psml.ring_gemm(ctx, A, B, out=C), reps)
                row[name + "_ms"] = ms
                row[name + "_useful_tops"] = pairs * 2.0 * n ** 3 / ms / 1e9
                if be == 2:
                    row["frac_of_int8_spec"] = row[name + "_useful_tops"] / INT8_DENSE_PEAK_TOPS
                ctx.close()
            # co-resident Beaver secure matmul (both parties: mask, open, Eq. 8 GEMM, trunc)
            ctx = psml.Ctx(l=l)
            As = psml.share(ring, 7, 1, A)
            Bs = psml.share(ring, 7, 2, B)
            U, V, Z = psml.triplet_gen(ctx, 3, 0, n, n, n)
            Cs = psml.empty_pair((n, n), l)
            ms = tev(lambda: psml.secure_matmul(ctx, As, Bs, U, V, Z, n, n, n, trunc=13, out=Cs), reps)
            row["beaver_ms"] = ms
            row["beaver_useful_tops"] = 2 * 2 * pairs * 2.0 * n ** 3 / ms / 1e9   # 2 parties x K' = 2K
            ctx.close()
            if n <= 2048:
                An, Bn = A.cpu().numpy(), B.cpu().numpy()
                t0 = time.perf_counter()
                W = orc.ring_matmul(An, Bn, l)
                oracle_t[(n, l)] = time.perf_counter() - t0
                psml.ring_gemm(psml.Ctx(l=l, backend=2), A, B, out=C)
                row["bitexact_vs_oracle"] = bool(np.array_equal(C.cpu().numpy().astype(np.uint64), W))
                row["oracle_s"] = oracle_t[(n, l)]
            else:
                base = max(k for k in oracle_t if k[1] == l)
                row["oracle_s_extrapolated_n3"] = oracle_t[base] * (n / base[0]) ** 3
            row["oracle_threads"] = orc.num_threads()
            print(json.dumps(row), flush=True)



def cfg5_sharded(ns, world, rank):
    """Config 5 over `world` GPUs (bench.py --sweep under torchrun): M-row sharding of the n^3
    product over data-parallel pairs: pair r holds rows [r n / world, (r + 1) n / world)
    of A (and of U, Z: psml_triplet_gen_rows) and the whole B (and V), computes its C rows with no
    cross-pair collective; the plain ring GEMM and the co-resident Beaver secure matmul are both
    timed per rank with CUDA events (barrier + synchronize around), the max over ranks taken, and
    the aggregate useful TOPS = the whole n^3 product's limb ops / that time.  Rank 0 checks its
    row block bit-exactly against the CPU oracle for n <= 1024.  One JSON line per (n, l) on rank 0."""
    import numpy as np
    import torch
    import torch.distributed as dist
    from oracle import core as orc
    from paper_conf_icpp_chenzzzz020_b200 import psml
    for n in ns:
        if n % world:
            continue
        m = n // world
        r0 = rank * m
        for l in (64, 32):
            pairs = 36 if l == 64 else 10
            ring = psml.Ring(l, 13)
            A = psml.prg_fill(ring, 1, psml.tag("bA"), 0, m * n, offset=r0 * n).view(m, n)   # this pair's rows of A
            B = psml.prg_fill(ring, 1, psml.tag("bB"), 0, n * n).view(n, n)
            C = psml.empty(0, l, (m, n))
            reps = 5 if n >= 4096 else 10
            ctx = psml.Ctx(l=l)
            dist.barrier()
            ms = max_over_ranks(tev(lambda: psml.ring_gemm(ctx, A, B, out=C), reps), world)
            row = {"n": n, "l": l, "gpus": world, "sharding": "M rows over pairs (no cross-pair collective)",
                   "rows_per_gpu": m, "gemm_ms": ms, "gemm_useful_tops_aggregate": pairs * 2.0 * n ** 3 / ms / 1e9}
            As = psml.share(ring, 7, 1, A)
            Bs = psml.share(ring, 7, 2, B)
            U, V, Z = psml.triplet_gen_rows(ctx, 3, 0, n, r0, m, n, n)
            Cs = psml.empty_pair((m, n), l)
            dist.barrier()
            ms = max_over_ranks(tev(lambda: psml.secure_matmul(ctx, As, Bs, U, V, Z, m, n, n, trunc=13, out=Cs),
                                    reps), world)
            row["beaver_ms"] = ms
            row["beaver_useful_tops_aggregate"] = 2 * 2 * pairs * 2.0 * n ** 3 / ms / 1e9
            if n <= 1024 and rank == 0:
                W = orc.ring_matmul(A.cpu().numpy().astype(np.uint64), B.cpu().numpy().astype(np.uint64), l)
                row["bitexact_vs_oracle_rank0_rows"] = bool(np.array_equal(C.cpu().numpy().astype(np.uint64), W))
            ctx.close()
            if rank == 0:
                print(json.dumps(row), flush=True)
            torch.cuda.synchronize()


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


def cpu_baseline(budget_s=12.0):
    """The oracle as it stands on this host: whole secure MLP training steps (batch 128)."""
    import oracle
    oracle.build()
    t1, cores = oracle_steps(1, base=10000)
    n = max(2, min(60, int(budget_s / max(t1, 1e-3))))
    t, cores = oracle_steps(n, base=10001)
    out = {"value": BATCH * n / t, "unit": "samples/s", "cores": cores, "kind": "oracle",
           "sample": f"{n} full oracle secure MLP training steps (batch 128) on the host",
           "cpu_model": cpu_model(), "nproc": os.cpu_count()}
    # the same oracle on ONE host thread (nproc and 1 thread), a few steps in a
    # subprocess with OMP_NUM_THREADS=1
    try:
        code = ("import sys, json; sys.path.insert(0, %r); import bench; "
                "t, c = bench.oracle_steps(%d, base=10100); print(json.dumps([t, c]))" % (ROOT, 3))
        r = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, timeout=300,
                           env=dict(os.environ, OMP_NUM_THREADS="1"), cwd=ROOT)
        t1s, c1 = json.loads(r.stdout.strip().splitlines()[-1])
        out["one_thread"] = {"value": BATCH * 3 / t1s, "unit": "samples/s", "cores": c1,
                             "sample": "3 full oracle secure MLP training steps, OMP_NUM_THREADS=1"}
    except Exception as e:  # noqa: BLE001 -- reported, never fatal
        out["one_thread"] = {"unavailable": str(e)[:200]}
    return out


# ---------------------------------------------------------------------------------------------
# reference arm: the CPU oracle (oracle/protocol.py) on the same workload
# ---------------------------------------------------------------------------------------------
def oracle_steps(n_steps, base=0, task=None):
    import synth
    from oracle import core
    from oracle import protocol as OP
    task = task or TASK
    m = OP.Model(task, synth.init_weights(task))
    t0 = time.perf_counter()
    for s in range(n_steps):
        X, Y = synth.batch(task, base + s)
        OP.train_step(m, X, Y, base + s)
    return time.perf_counter() - t0, core.num_threads()


SECONDARY = (("linreg", "config 2: secure linear regression, MNIST-shaped, batch 128"),
             ("logreg", "config 2: secure logistic regression (Eq. 9), MNIST-shaped, batch 128"),
             ("cnn", "config 4: secure CNN (conv 5x5x16 im2col, FC 64, FC 10), CIFAR-shaped, batch 128"),
             ("svm", "SURVEY f4: secure linear SVM (hinge subgradient, DESIGN.md R24), MNIST-shaped, batch 128"),
             ("rnn", "SURVEY f4: secure Elman RNN (T = 16, BPTT, DESIGN.md R25), synthetic sequences, batch 128"))


def secondary_figures(K=50):
    """The other BASELINE configs / workloads on the same GPU, each as its own pipelined CUDA graph
    (client share + next step's dealer + online step + update), K timed steps after a warm-up, CUDA
    events with the 256 MiB L2 flush between steps; secure inference (forward half + its dealer);
    beside the oracle timed on the host (a few whole steps; 1 for the CNN)."""
    import torch
    import synth
    from paper_conf_icpp_chenzzzz020_b200.train import SecureTrainer
    dev = torch.device("cuda")
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream()
    out = {}
    for task, what in SECONDARY:
        try:
            tr = SecureTrainer(task, synth.init_weights(task))
            data = [synth.batch(task, s) for s in range(8)]
            Xs = [torch.from_numpy(x).to(dev) for x, _ in data]
            Ys = [torch.from_numpy(y).to(dev) for _, y in data]
            tr.step(Xs[0], Ys[0], 0)
            tr.capture(pipelined=True)

            def timed(fn, n, base):
                evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(n)]
                torch.cuda.synchronize()
                for i in range(n):
                    flush.zero_()
                    evs[i][0].record(stream)
                    fn(base + i)
                    evs[i][1].record(stream)
                torch.cuda.synchronize()
                return sum(a.elapsed_time(b) for a, b in evs) / 1e3
            timed(lambda s: tr.graph_step(Xs[s % 8], Ys[s % 8], s), 3, 1)
            n = K if task != "cnn" else max(10, K // 4)
            t = timed(lambda s: tr.graph_step(Xs[s % 8], Ys[s % 8], s), n, 4)

            def infer(s):
                Xsh, _ = tr.share_batch(Xs[s % 8], Ys[s % 8], s)
                tr.infer_shares(Xsh, s)
            ti = timed(infer, n, 100000)
            tr.close()
            n_or = 1 if task == "cnn" else 5
            t_or, cores = oracle_steps(n_or, base=20000, task=task)
            out[task] = {"config": what, "samples_per_s": 128 * n / t, "ms_per_step": 1e3 * t / n,
                         "infer_samples_per_s": 128 * n / ti, "steps": n,
                         "cpu_baseline": {"value": 128 * n_or / t_or, "unit": "samples/s", "cores": cores,
                                          "kind": "oracle", "sample": f"{n_or} whole oracle training step(s)"}}
        except Exception as e:   # noqa: BLE001 -- reported, never fatal to the headline line
            out[task] = {"config": what, "error": str(e)[:300]}
    return out


def arm_config(world, scaling="weak"):
    """The `config` of both arms' JSON lines."""
    strong = scaling == "strong" and world > 1
    return {"workload": WORKLOAD, "global_batch": BATCH if strong else BATCH * world,
            "per_pair_batch": BATCH // world if strong else BATCH,
            "ring": "Z_2^64, 13 fractional bits", "parallelism": f"dp{world} (pairs)",
            "l2": "256 MiB flush between timed steps (outside the events)",
            "step": "client encode+share, dealer (offline), online secure step"}


def bench_reference(args, budget_s=150.0):
    """The oracle as it stands on the host cores (rank 0 only).  W warm-up steps (at most 3),
    then min(K, what fits in ~budget_s) whole oracle training steps of the same workload, so
    the run ends within a few minutes whatever K is; the step count is stated in `sample`."""
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return None
    import oracle
    oracle.build()
    tw, _ = oracle_steps(max(1, min(args.warmup, 3)))
    t1 = tw / max(1, min(args.warmup, 3))
    n = max(1, min(args.steps, int(budget_s / max(t1, 1e-3))))
    t, cores = oracle_steps(n, base=args.warmup)
    v = BATCH * n / t   # the oracle simulates one pair on the host, whatever N
    return {
        "impl": "reference", "metric": METRIC, "value": v, "unit": "samples/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * t / n,
        "higher_is_better": True, "scaling": "strong" if (args.scaling == "strong" and world > 1) else "weak",
        "vs_baseline": None, "dtype": "u64",
        "data": ("synthetic (CIFAR-shaped 3x32x32 8-bit pixels; teacher-CNN labels)" if TASK == "cnn" else
                 "synthetic (MNIST-shaped 8-bit pixels, 81% zeros; teacher labels)"),
        "config": arm_config(world, args.scaling),
        "cpu_baseline": {"value": v, "unit": "samples/s", "cores": cores, "kind": "oracle", "cpu_model": cpu_model(),
                         "sample": f"{n} of the {args.steps} requested steps: full oracle secure training "
                                   f"steps of batch {BATCH} (both parties simulated) on the host"},
        "e2e": {"value": v, "unit": "samples/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }


def main():
    args = parse()
    if args.impl == "reference":
        out = bench_reference(args)
        if out is not None:
            print(json.dumps(out), flush=True)
        return
    if args.sweep:
        from paper_conf_icpp_chenzzzz020_b200 import build
        build.build()
        ns = [int(x) for x in args.sweep.split(",")]
        if int(os.environ.get("WORLD_SIZE", "1")) > 1:
            world, rank, _ = dist_setup(args)
            cfg5_sharded(ns, world, rank)
        else:
            cfg5_sweep(ns)
        return
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if args.deployment == "split" or (args.deployment == "auto" and world >= 2):
        result, rank = bench_split(args)
        if rank == 0:
            print(json.dumps(result), flush=True)
        return
    result, tr, world, rank = bench_ours(args)
    if TASK != "mlp":
        result["metric"] = f"secure {TASK} training samples/s (secondary config; headline metric is the MLP)"
    if rank == 0 and world == 1 and not args.no_ring_gemm:
        result["ring_gemm"] = [ring_gemm_figure(4096, 64), ring_gemm_figure(4096, 32),
                               ring_gemm_figure(1024, 64, reps=20), ring_gemm_figure(1024, 32, reps=20),
                               ring_gemm_figure(512, 64, reps=20)]
        result["beaver_matmul_cfg1"] = beaver_latency_figure()
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        result["cpu_baseline"] = cpu_baseline()
    if rank == 0 and world == 1 and not args.no_secondary:
        result["secondary_configs"] = secondary_figures()
    if rank == 0:
        print(json.dumps(result), flush=True)


if __name__ == "__main__":
    main()
