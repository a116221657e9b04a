#!/bin/bash
# GPU-box job: compile-time variants of tc_seg on the stand-alone small products (tools/tc_small_ab.py)
# and the headline bench.  Usage: ab_tcseg.sh "<flags A>" "<flags B>" ...
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
i=0
for flags in "$@"; do
  PSML_NVCC_EXTRA="$flags" python -m paper_conf_icpp_chenzzzz020_b200.build --force > gpurun_out/abt_build$i.log 2>&1 || { echo "build $i failed"; continue; }
  echo "=== [$flags]"
  timeout 300 python tools/tc_small_ab.py 512,1024,2048 64,32 2>/dev/null | grep '"tc_small": 2' | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l); print('  n', d['n'], 'l', d['l'], 'plain_us', round(d['plain_ms']*1e3,1), 'beaver_us', round(d['beaver_ms']*1e3,1))"
  timeout 600 python bench.py --steps 500 --no-ring-gemm --no-cpu-baseline --no-secondary > gpurun_out/abt$i.json 2>/dev/null
  python -c "
import json; d=json.load(open('gpurun_out/abt$i.json')); k=d.get('kernel_classes',{})
print('  value', round(d['value']), 'e2e', round(d['e2e']['value']), 'online_graph', round(d['online_graph_samples_per_s']), 'tc', round(k['ring_gemm_tcgen05']['ms_per_step']*1e3,1))"
  i=$((i+1))
done
python -m paper_conf_icpp_chenzzzz020_b200.build --force > /dev/null 2>&1
