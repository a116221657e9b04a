cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_primitives.py -x -q -k "secure_matmul or encode" 2>&1 | tail -2
timeout 900 python -m pytest tests/test_gpu_training.py tests/test_gpu_split.py -x -q 2>&1 | tail -2
timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-ring-gemm > gpurun_out/b57.json 2> gpurun_out/b57.err
tail -2 gpurun_out/b57.err
python -c "
import json; d=json.load(open('gpurun_out/b57.json'))
print('value',round(d['value']),'online_graph',round(d.get('online_graph_samples_per_s')),'e2e',round(d['e2e']['value']),'ms',round(d['ms_per_step'],4)); print({k:(round(v['ms_per_step'],4), v['launches_per_step']) for k,v in d['kernel_classes'].items()}); print(d['roofline'])"
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches57_graph.csv python tools/step_profile.py mlp 4 > gpurun_out/ncu57b.log 2>&1
