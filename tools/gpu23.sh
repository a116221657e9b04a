cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q -x -k "not one_epoch" 2>&1 | tail -3
timeout 600 python bench.py --no-cpu-baseline --no-ring-gemm > gpurun_out/bench10.json 2> gpurun_out/bench10.err
tail -2 gpurun_out/bench10.err
python -c "
import json; d=json.load(open('gpurun_out/bench10.json'))
print('value',round(d['value']),'online',round(d['online_samples_per_s']),'eager',round(d['eager_samples_per_s']),'e2e',round(d['e2e']['value']),'ms',d['ms_per_step'], d['clocks'])
for k,v in d['kernel_classes'].items(): print(k, round(v['ms_per_step'],4), round(v['ms_per_launch'],4), v['launches_per_step'])
print(d['roofline'])"
