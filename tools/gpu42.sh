cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_primitives.py tests/test_gpu_training.py tests/test_gpu_split.py -q -x -k "not one_epoch" 2>&1 | tail -4
timeout 120 python tools/gemm_lat.py 1
timeout 300 python bench.py --steps 2000 --no-cpu-baseline --no-ring-gemm > gpurun_out/b42.json 2> gpurun_out/b42.err
tail -2 gpurun_out/b42.err
python -c "
import json; d=json.load(open('gpurun_out/b42.json'))
print('value',d['value'],'online_graph',d.get('online_graph_samples_per_s'),'online',d['online_samples_per_s'],'e2e',d['e2e']['value'],'ms',d['ms_per_step'],'nodes',d['gpu_launches'])
for k,v in d['kernel_classes'].items(): print(k, round(v['ms_per_step'],4), round(v['ms_per_launch'],4), v['launches_per_step'])"
