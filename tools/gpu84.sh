cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_training.py -x -q -k "cnn or backends" 2>&1 | tail -2
timeout 900 python bench.py --task cnn --steps 150 --no-cpu-baseline --no-ring-gemm > gpurun_out/b84c.json 2> gpurun_out/b84c.err
python -c "
import json; d=json.load(open('gpurun_out/b84c.json'))
print('cnn value',round(d['value']),'e2e',round(d['e2e']['value']),'online',round(d['online_samples_per_s']),'infer',round(d['infer_samples_per_s']),'ms',round(d['ms_per_step'],4)); print({k:(round(v['ms_per_step'],4), v['launches_per_step']) for k,v in d['kernel_classes'].items()})"
run() {
  timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-ring-gemm > gpurun_out/b84.json 2> gpurun_out/b84.err
  python -c "
import json; d=json.load(open('gpurun_out/b84.json'))
print('$1 value',round(d['value']),'e2e',round(d['e2e']['value']),'online_graph',round(d['online_graph_samples_per_s']),'ms',round(d['ms_per_step'],4), d['clocks']['sm_mhz'], 'dealer', round(d['kernel_classes']['dealer']['ms_per_step']*1e3,1))" 2>&1 | tail -1
}
run "TILE=32"
PSML_DEAL_TILE=64 run "TILE=64"
run "TILE=32 again"
PSML_DEAL_TILE=64 run "TILE=64 again"
