cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
run() {
  timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-ring-gemm > gpurun_out/b96.json 2> gpurun_out/b96.err
  python -c "
import json; d=json.load(open('gpurun_out/b96.json'))
print('$1 value',round(d['value']),'e2e',round(d['e2e']['value']),'ms',round(d['ms_per_step'],4), d['clocks']['sm_mhz'])" 2>&1 | tail -1
}
run "default"
PSML_DEAL_AFTER=2 run "AFTER=2"
PSML_DEAL_KS=8 run "KS=8"
PSML_DEAL_KS=2 run "KS=2"
PSML_DEAL_AFTER=0 run "AFTER=0"
run "default again"
