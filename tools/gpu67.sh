cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_training.py tests/test_gpu_split.py tests/test_gpu_primitives.py -x -q 2>&1 | tail -2
timeout 900 python bench.py --task cnn --steps 150 --no-cpu-baseline --no-ring-gemm > gpurun_out/b67c.json 2> gpurun_out/b67c.err
python -c "
import json; d=json.load(open('gpurun_out/b67c.json'))
print('cnn value',round(d['value']),'online',round(d['online_samples_per_s']),'infer',round(d['infer_samples_per_s']),'ms',round(d['ms_per_step'],4)); print({k:(round(v['ms_per_step'],4), v['launches_per_step']) for k,v in d['kernel_classes'].items()})"
for cfg in "4 8" "4 0" "8 4"; do
set -- $cfg
PSML_DEAL_KS=$1 PSML_DEAL_CTAS=$2 timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-ring-gemm > gpurun_out/b67.json 2> gpurun_out/b67.err
python -c "
import json; d=json.load(open('gpurun_out/b67.json'))
print('KS=$1 CTAS=$2 value',round(d['value']),'online_graph',round(d.get('online_graph_samples_per_s')),'ms',round(d['ms_per_step'],4))"
done
for c in 8 0; do
PSML_DEAL_CTAS=$c timeout 900 python bench.py --task cnn --steps 100 --no-cpu-baseline --no-ring-gemm > gpurun_out/b67c.json 2> gpurun_out/b67c.err
python -c "
import json; d=json.load(open('gpurun_out/b67c.json'))
print('cnn CTAS=$c value',round(d['value']),'online',round(d['online_samples_per_s']),'ms',round(d['ms_per_step'],4))"
done
