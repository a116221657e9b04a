cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q -x -k "not one_epoch and not fullsize and not split" 2>&1 | tail -2
for i in 1 2; do timeout 600 python bench.py --no-cpu-baseline --no-ring-gemm > gpurun_out/bench11.json 2>/dev/null
python -c "
import json; d=json.load(open('gpurun_out/bench11.json'))
print('value',round(d['value']),'online',round(d['online_samples_per_s']),'e2e',round(d['e2e']['value']),'ms',round(d['ms_per_step'],4))
for k,v in d['kernel_classes'].items(): print(k, round(v['ms_per_step'],4), round(v['ms_per_launch'],4), v['launches_per_step'])"; done
