cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests/test_gpu_training.py -q -x -k "graph or bitexact" 2>&1 | tail -5
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench4.json 2> gpurun_out/bench4.err
tail -3 gpurun_out/bench4.err
python -c "
import json; d=json.load(open('gpurun_out/bench4.json'))
print('value',d['value'],'online',d['online_samples_per_s'],'eager',d['eager_samples_per_s'],'e2e',d['e2e']['value'],'ms',d['ms_per_step'],d['clocks'],'launches',d['gpu_launches'],d['cuda_graph']['kernel_nodes_per_step'])
for k,v in d['kernel_classes'].items(): print(k, round(v['ms_per_step'],4), round(v['ms_per_launch'],4), v['launches_per_step'])
print(d['roofline'])"
