cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
run() {
  timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-ring-gemm > gpurun_out/b73.json 2> gpurun_out/b73.err
  python -c "
import json; d=json.load(open('gpurun_out/b73.json'))
print('$1 value',round(d['value']),'e2e',round(d['e2e']['value']),'ms',round(d['ms_per_step'],4), d['clocks']['sm_mhz'], 'offline ms', round(d['offline']['ms_per_step'],4))" 2>&1 | tail -1
}
run "SPLIT=1 AFTER=1"
PSML_DEAL_SPLIT=0 run "SPLIT=0 AFTER=1"
PSML_DEAL_AFTER=2 run "SPLIT=1 AFTER=2"
PSML_DEAL_CTAS=2 run "SPLIT=1 CTAS=2"
PSML_DEAL_CTAS=3 run "SPLIT=1 CTAS=3"
run "SPLIT=1 AFTER=1 again"
PSML_DEAL_SPLIT=0 run "SPLIT=0 AFTER=1 again"
timeout 300 python tools/timeline.py mlp 20 gpurun_out/timeline_mlp3.json 2>&1 | tail -24
( time timeout 1500 python -m pytest tests/test_gpu_training.py -x -q ) 2>&1 | tail -4
