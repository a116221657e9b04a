cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_training.py -x -q -k "bitexact or graph" 2>&1 | tail -1
PSML_DEALER_PRE=3 timeout 900 python -m pytest tests/test_gpu_training.py -x -q -k "bitexact or graph" 2>&1 | tail -1
run() {
  timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-ring-gemm > gpurun_out/b82.json 2> gpurun_out/b82.err
  python -c "
import json; d=json.load(open('gpurun_out/b82.json'))
print('$1 value',round(d['value']),'e2e',round(d['e2e']['value']),'online_graph',round(d['online_graph_samples_per_s']),'ms',round(d['ms_per_step'],4), d['clocks']['sm_mhz'], {k:round(v['ms_per_step']*1e3,1) for k,v in d['kernel_classes'].items()})" 2>&1 | tail -1
}
for v in 0 1 2 3 0 2; do PSML_DEALER_PRE=$v run "PRE=$v"; done
