#!/bin/bash
# GPU-box job: the config-5 M-row sharded sweep (bench.py --sweep under torchrun) with all N ranks
# on the one GPU over gloo -- a functional / parity check of the sharded path on a 1-GPU lease (the
# ranks time-share one GPU, so the TOPS are not a multi-GPU figure).  Usage: sweep_sharded_shared.sh [N] [sizes]
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
N=${1:-2}; NS=${2:-512,1024}
PSML_SHARE_GPU=1 PSML_DIST_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node $N \
  --master-addr 127.0.0.1 --master-port 29535 bench.py --gpus $N --sweep $NS > gpurun_out/sweep_sharded$N.jsonl \
  2> gpurun_out/sweep_sharded$N.err
echo "rc=$?"; tail -2 gpurun_out/sweep_sharded$N.err; cat gpurun_out/sweep_sharded$N.jsonl
