cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
run() {
  timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-ring-gemm > gpurun_out/b74.json 2> gpurun_out/b74.err
  python -c "
import json; d=json.load(open('gpurun_out/b74.json'))
print('$1 value',round(d['value']),'e2e',round(d['e2e']['value']),'online_graph',round(d['online_graph_samples_per_s']),'ms',round(d['ms_per_step'],4), d['clocks']['sm_mhz'])" 2>&1 | tail -1
}
run "GW=1"
PSML_GRADW_BRANCH=0 run "GW=0"
run "GW=1 again"
PSML_GRADW_BRANCH=0 run "GW=0 again"
timeout 300 python tools/timeline.py mlp 20 gpurun_out/timeline_mlp4.json 2>&1 | tail -24
timeout 1500 python -m pytest tests/test_gpu_training.py -x -q 2>&1 | tail -2
