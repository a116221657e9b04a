cd $GRAFT_REPO_ROOT
for mode in fused rounds fused rounds; do
  PSML_OPEN=$mode timeout 600 python bench.py --no-cpu-baseline --no-ring-gemm > gpurun_out/ab_$mode.json 2>/dev/null
  python -c "
import json; d=json.load(open('gpurun_out/ab_$mode.json'))
print('$mode', round(d['value']),'online',round(d['online_samples_per_s']),'e2e',round(d['e2e']['value']),'ms',round(d['ms_per_step'],4))"
done
