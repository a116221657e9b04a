cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_training.py -x -q -k "graph or bench_path" 2>&1 | tail -1
run() {
  timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-ring-gemm > gpurun_out/b92.json 2> gpurun_out/b92.err
  python -c "
import json; d=json.load(open('gpurun_out/b92.json'))
print('$1 value',round(d['value']),'e2e',round(d['e2e']['value']),'online_graph',round(d['online_graph_samples_per_s']),'ms',round(d['ms_per_step'],4), d['clocks']['sm_mhz'])" 2>&1 | tail -1
}
run "order-swap CTAS2=4"
PSML_DEAL_CTAS2=3 run "CTAS2=3"
PSML_DEAL_CTAS2=2 run "CTAS2=2"
PSML_DEAL_CTAS=6 PSML_DEAL_CTAS2=2 run "CTAS=6 CTAS2=2"
PSML_DEAL_CTAS=8 PSML_DEAL_CTAS2=3 run "CTAS=8 CTAS2=3"
run "order-swap again"
timeout 300 python tools/timeline.py mlp 20 gpurun_out/timeline_92.json 2>&1 | tail -27
