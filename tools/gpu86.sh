cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
PSML_MSB_TPB=64 timeout 900 python -m pytest tests/test_gpu_training.py -x -q -k "bitexact or graph" 2>&1 | tail -1
run() {
  timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-ring-gemm > gpurun_out/b86.json 2> gpurun_out/b86.err
  python -c "
import json; d=json.load(open('gpurun_out/b86.json'))
print('$1 value',round(d['value']),'e2e',round(d['e2e']['value']),'online_graph',round(d['online_graph_samples_per_s']),'ms',round(d['ms_per_step'],4), d['clocks']['sm_mhz'], 'msb', round(d['kernel_classes']['msb_relu_eq9_rounds']['ms_per_step']*1e3,1))" 2>&1 | tail -1
}
for t in 256 128 64 32 256 64; do PSML_MSB_TPB=$t run "TPB=$t"; done
