#!/bin/bash
# GPU-box job: compile-time variants on the CNN (config 4) bench line.  Usage: ab_cnn.sh "<flags A>" ...
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
i=0
for flags in "$@"; do
  PSML_NVCC_EXTRA="$flags" python -m paper_conf_icpp_chenzzzz020_b200.build --force > gpurun_out/abc_build$i.log 2>&1 || { echo "build $i failed"; continue; }
  timeout 600 python bench.py --task cnn --steps 30 --no-ring-gemm --no-cpu-baseline --no-secondary > gpurun_out/abc$i.json 2>/dev/null
  python -c "
import json; d=json.load(open('gpurun_out/abc$i.json')); k=d.get('kernel_classes',{})
print('[$flags]', 'value', round(d['value']), 'e2e', round(d['e2e']['value']), {c: round(v['ms_per_step']*1e3,1) for c, v in k.items() if c != '_check'})"
  i=$((i+1))
done
python -m paper_conf_icpp_chenzzzz020_b200.build --force > /dev/null 2>&1
