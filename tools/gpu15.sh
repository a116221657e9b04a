cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests -m gpu -q -x -k "not one_epoch" 2>&1 | tail -3
timeout 600 python bench.py --no-cpu-baseline --no-ring-gemm > gpurun_out/bench6.json 2> gpurun_out/bench6.err
tail -2 gpurun_out/bench6.err
python -c "
import json; d=json.load(open('gpurun_out/bench6.json'))
print('value',d['value'],'online',d['online_samples_per_s'],'eager',d['eager_samples_per_s'],'e2e',d['e2e']['value'],'ms',d['ms_per_step'], d['cuda_graph']['kernel_nodes_per_step'])
for k,v in d['kernel_classes'].items(): print(k, round(v['ms_per_step'],4), round(v['ms_per_launch'],4), v['launches_per_step'])
print(d['roofline'])"
