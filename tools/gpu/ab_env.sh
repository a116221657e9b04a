#!/bin/bash
# GPU-box job: A/B of psml_options (via the binding's PSML_* environment overrides) on the headline
# bench.  Usage: ab_env.sh "<VAR=val ...>" "<VAR=val ...>" ...   ("" = defaults); each run 500 steps.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
i=0
for envs in "$@"; do
  env $envs timeout 600 python bench.py --steps 500 --no-ring-gemm --no-cpu-baseline --no-secondary --no-classes > gpurun_out/abe$i.json 2>gpurun_out/abe$i.err
  python -c "
import json; d=json.load(open('gpurun_out/abe$i.json'))
print('[$envs]', 'value', round(d['value']), 'e2e', round(d['e2e']['value']), 'online_graph', round(d['online_graph_samples_per_s']))" || tail -3 gpurun_out/abe$i.err
  i=$((i+1))
done
