cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
run() {
  timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-ring-gemm > gpurun_out/b100.json 2> gpurun_out/b100.err
  python -c "
import json; d=json.load(open('gpurun_out/b100.json'))
print('$1 value',round(d['value']),'e2e',round(d['e2e']['value']),'ms',round(d['ms_per_step'],4), d['clocks']['sm_mhz'])" 2>&1 | tail -1
}
python -c "import torch; print(torch.cuda.Stream.priority_range())"
run "default"
PSML_DEAL_PRIO1=1 run "PRIO1=1"
PSML_DEAL_PRIO1=2 run "PRIO1=2"
PSML_DEAL_PRIO1=3 run "PRIO1=3"
run "default again"
