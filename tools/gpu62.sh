cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_primitives.py -x -q 2>&1 | tail -2
timeout 1200 python -m pytest tests/test_gpu_training.py tests/test_gpu_split.py -x -q 2>&1 | tail -2
for t in cnn mlp; do
timeout 900 python bench.py --task $t --steps 200 --no-cpu-baseline --no-ring-gemm > gpurun_out/b62_$t.json 2> gpurun_out/b62_$t.err
tail -1 gpurun_out/b62_$t.err
python -c "
import json; d=json.load(open('gpurun_out/b62_$t.json'))
print('$t value',round(d['value']),'online',round(d['online_samples_per_s']),'infer',round(d['infer_samples_per_s']),'e2e',round(d['e2e']['value']),'ms',round(d['ms_per_step'],4)); print({k:(round(v['ms_per_step'],4), v['launches_per_step']) for k,v in d['kernel_classes'].items()})"
done
