#!/bin/bash
# GPU-box job: A/B of compile-time variants on the headline bench (no ncu, no cpu baseline).
# Usage: ab_build.sh "<nvcc -D flags A>" "<flags B>" ...   ("" = the default build)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
i=0
for flags in "$@"; do
  PSML_NVCC_EXTRA="$flags" python -m paper_conf_icpp_chenzzzz020_b200.build --force > gpurun_out/ab_build$i.log 2>&1 || { echo "build $i failed"; tail -5 gpurun_out/ab_build$i.log; continue; }
  timeout 600 python bench.py --steps 500 --no-ring-gemm --no-cpu-baseline --no-secondary > gpurun_out/ab$i.json 2>/dev/null
  python -c "
import json; d=json.load(open('gpurun_out/ab$i.json')); k=d.get('kernel_classes',{})
print('[$flags]', 'value', round(d['value']), 'e2e', round(d['e2e']['value']), 'online_graph', round(d['online_graph_samples_per_s']),
      {c: round(v['ms_per_step']*1e3,1) for c, v in k.items() if c != '_check'})"
  i=$((i+1))
done
