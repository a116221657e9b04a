cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_primitives.py -x -q -k "secure_matmul" 2>&1 | tail -5
timeout 600 python -m pytest tests/test_gpu_training.py -x -q 2>&1 | tail -5
timeout 300 python bench.py --steps 500 --no-cpu-baseline --no-ring-gemm > gpurun_out/b48.json 2> gpurun_out/b48.err
tail -2 gpurun_out/b48.err
python -c "
import json; d=json.load(open('gpurun_out/b48.json'))
print('value',round(d['value']),'online_graph',round(d.get('online_graph_samples_per_s')),'e2e',round(d['e2e']['value']),'ms',round(d['ms_per_step'],4)); print(json.dumps(d['kernel_classes'], indent=0))"
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches48_graph.csv python tools/step_profile.py mlp 4 > gpurun_out/ncu48b.log 2>&1
tail -1 gpurun_out/ncu48b.log
