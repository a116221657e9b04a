cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_training.py tests/test_gpu_primitives.py tests/test_gpu_split.py -x -q 2>&1 | tail -2
for r in 1 2; do
timeout 900 python bench.py --no-cpu-baseline --no-ring-gemm > gpurun_out/b90.json 2> gpurun_out/b90.err
python -c "
import json; d=json.load(open('gpurun_out/b90.json'))
print('value',round(d['value']),'e2e',round(d['e2e']['value']),'online_graph',round(d['online_graph_samples_per_s']),'ms',round(d['ms_per_step'],4), d['clocks']['sm_mhz'], {k:round(v['ms_per_step']*1e3,1) for k,v in d['kernel_classes'].items()})"
done
