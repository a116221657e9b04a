#!/bin/bash
# GPU-box job: bench.py --gpus N --deployment coresident --scaling strong with all N ranks on the one
# GPU over gloo (N co-resident pairs, one global batch of 128 rows) -- a functional check
# of the strong-scaling bench path on a 1-GPU lease, not a performance configuration.
# Usage: bench_strong_shared.sh [N] [steps]
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
N=${1:-2}; K=${2:-20}
PSML_SHARE_GPU=1 PSML_DIST_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node $N \
  --master-addr 127.0.0.1 --master-port 29534 bench.py --gpus $N --deployment coresident --scaling strong \
  --steps $K --warmup 3 > gpurun_out/bench_strong$N.json 2> gpurun_out/bench_strong$N.err
echo "rc=$?"; tail -3 gpurun_out/bench_strong$N.err; python -c "
import json; d=json.load(open('gpurun_out/bench_strong$N.json'))
print('N=$N', d['scaling'], 'value', round(d['value']), 'ms/step', round(d['ms_per_step'],3), d['config']['global_batch'], d['config']['per_pair_batch'])"
