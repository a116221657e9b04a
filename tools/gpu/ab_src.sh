#!/bin/bash
# GPU-box job: A/B of a source-file variant on the headline bench.  Usage: ab_src.sh <repo path> <variant file> [rounds]
# Alternates (current tree, variant) `rounds` times; restores the current file at the end.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
dst=$1; alt=$2; n=${3:-2}
cp "$dst" /tmp/ab_cur_src
for r in $(seq 1 $n); do
  for v in cur alt; do
    if [ $v = cur ]; then cp /tmp/ab_cur_src "$dst"; else cp "$alt" "$dst"; fi
    python -m paper_conf_icpp_chenzzzz020_b200.build --force > gpurun_out/ab_src_build.log 2>&1 || { echo "build $v failed"; tail -5 gpurun_out/ab_src_build.log; continue; }
    timeout 600 python bench.py --steps 500 --no-ring-gemm --no-cpu-baseline --no-secondary > gpurun_out/ab_src_$v$r.json 2>/dev/null
    python -c "
import json; d=json.load(open('gpurun_out/ab_src_$v$r.json')); k=d.get('kernel_classes',{})
print('[$v]', 'value', round(d['value']), 'e2e', round(d['e2e']['value']), 'online_graph', round(d['online_graph_samples_per_s']),
      {c: round(v['ms_per_step']*1e3,1) for c, v in k.items() if c != '_check'})"
  done
done
cp /tmp/ab_cur_src "$dst"
python -m paper_conf_icpp_chenzzzz020_b200.build --force > /dev/null 2>&1
