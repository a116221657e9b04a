#!/bin/bash
# GPU-box job: bench.py --gpus 2 (split deployment) with both ranks on the one GPU over gloo --
# exercises the multi-rank bench path on a 1-GPU lease (not a performance configuration).
# Usage: bench2_shared.sh [steps] [extra bench args...]
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
K=${1:-20}; shift
TAG=$(echo "$*" | tr -d ' -')
PSML_SHARE_GPU=1 PSML_DIST_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
  --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps $K --warmup 3 "$@" \
  > gpurun_out/bench2_shared$TAG.json 2> gpurun_out/bench2_shared$TAG.err
echo "rc=$?"; python -c "
import json; d=json.load(open('gpurun_out/bench2_shared$TAG.json'))
print('$*', 'ms/step', round(d['ms_per_step'],2), 'exchanges/step', d['exchanges_per_step'], 'bytes/step/party', d['bytes_sent_per_step_per_party'])"
