cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
run() {
  timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-ring-gemm > gpurun_out/b75.json 2> gpurun_out/b75.err
  python -c "
import json; d=json.load(open('gpurun_out/b75.json'))
print('$1 value',round(d['value']),'e2e',round(d['e2e']['value']),'online_graph',round(d['online_graph_samples_per_s']),'ms',round(d['ms_per_step'],4), d['clocks']['sm_mhz'], 'tc', round(d['kernel_classes']['ring_gemm_tcgen05']['ms_per_step']*1e3,1))" 2>&1 | tail -1
}
run "FILL=2"
PSML_TCSEG_FILL=1 run "FILL=1"
run "FILL=2 again"
PSML_TCSEG_FILL=1 run "FILL=1 again"
