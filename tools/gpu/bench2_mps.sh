#!/bin/bash
# GPU-box job: bench.py --gpus 2 (split deployment: party 0 and party 1 in two processes) on the one
# leased GPU under MPS, so the two parties' kernels run concurrently (without MPS the processes
# time-slice and every exchange waits for a context switch).  Both parties share the GPU's SMs and
# HBM, and the peer-memory exchanges go through the same HBM instead of NVLink.
# Usage: bench2_mps.sh [steps] [extra bench args...]
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
export CUDA_MPS_PIPE_DIRECTORY=/tmp/psml_mps_pipe CUDA_MPS_LOG_DIRECTORY=/tmp/psml_mps_log
mkdir -p $CUDA_MPS_PIPE_DIRECTORY $CUDA_MPS_LOG_DIRECTORY
nvidia-cuda-mps-control -d || { echo "MPS unavailable"; exit 1; }
K=${1:-50}; shift
TAG=$(echo "$*" | tr -d ' -')
PSML_SHARE_GPU=1 PSML_DIST_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
  --master-addr 127.0.0.1 --master-port 29534 bench.py --gpus 2 --steps $K --warmup 5 "$@" \
  > gpurun_out/bench2_mps$TAG.json 2> gpurun_out/bench2_mps$TAG.err
rc=$?
echo quit | nvidia-cuda-mps-control
echo "rc=$rc"; python -c "
import json; d=json.load(open('gpurun_out/bench2_mps$TAG.json'))
print('MPS $*', 'samples/s', round(d['value']), 'ms/step', round(d['ms_per_step'],3), 'e2e', round(d['e2e']['value']), 'exchanges/step', d['exchanges_per_step'], 'bytes/step/party', d['bytes_sent_per_step_per_party'])" || tail -20 gpurun_out/bench2_mps$TAG.err
