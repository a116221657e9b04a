#!/bin/bash
# GPU-box job: bench.py --gpus 2 (split deployment) with both ranks on the one GPU over gloo --
# exercises the multi-rank bench path on a 1-GPU lease (not a performance configuration).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
PSML_SHARE_GPU=1 PSML_DIST_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
  --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps ${1:-20} --warmup 3 \
  > gpurun_out/bench2_shared.json 2> gpurun_out/bench2_shared.err
echo "rc=$?"; tail -c 3000 gpurun_out/bench2_shared.json; tail -5 gpurun_out/bench2_shared.err
