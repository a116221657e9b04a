cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_training.py -x -q -k "step_host or bench_path" 2>&1 | tail -1
for r in 1 2; do
timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-ring-gemm > gpurun_out/b97.json 2> gpurun_out/b97.err
python -c "
import json; d=json.load(open('gpurun_out/b97.json'))
print('value',round(d['value']),'e2e',round(d['e2e']['value']),'ms',round(d['ms_per_step'],4), d['clocks']['sm_mhz'])"
done
