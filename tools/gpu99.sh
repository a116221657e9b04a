cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
run() {
  timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-ring-gemm > gpurun_out/b99.json 2> gpurun_out/b99.err
  python -c "
import json; d=json.load(open('gpurun_out/b99.json'))
print('$1 value',round(d['value']),'e2e',round(d['e2e']['value']),'ms',round(d['ms_per_step'],4), d['clocks']['sm_mhz'])" 2>&1 | tail -1
}
run "default"
PSML_GRADW_BRANCH=0 run "GRADW_BRANCH=0"
PSML_SEG=simt run "SEG=simt"
PSML_PRIO=0 run "PRIO=0"
PSML_DEAL_SPLIT=0 run "DEAL_SPLIT=0"
run "default again"
