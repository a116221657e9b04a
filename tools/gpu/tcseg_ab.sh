#!/bin/bash
# A/B of the step's tcgen05 product route: in-kernel split (default) vs limb planes + v4 (PSML_TCSEG=1)
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
for v in 0 1; do
  PSML_TCSEG=$v timeout 600 python bench.py --steps 300 --no-ring-gemm --no-cpu-baseline > gpurun_out/tcseg$v.json 2>/dev/null
  python -c "
import json; d=json.load(open('gpurun_out/tcseg$v.json'))
k=d.get('kernel_classes',{})
print('TCSEG=$v value',round(d['value']),'online_graph',round(d['online_graph_samples_per_s']),'tc ms/launch',k.get('ring_gemm_tcgen05',{}).get('ms_per_launch'),'tc ms/step',k.get('ring_gemm_tcgen05',{}).get('ms_per_step'))"
done
