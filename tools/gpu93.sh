cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
run() {
  timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-ring-gemm > gpurun_out/b93.json 2> gpurun_out/b93.err
  python -c "
import json; d=json.load(open('gpurun_out/b93.json'))
print('$1 value',round(d['value']),'e2e',round(d['e2e']['value']),'online_graph',round(d['online_graph_samples_per_s']),'ms',round(d['ms_per_step'],4), d['clocks']['sm_mhz'])" 2>&1 | tail -1
}
run "default (CTAS2=2)"
PSML_DEAL_CTAS2=1 run "CTAS2=1"
PSML_DEAL_CTAS=3 run "CTAS=3 CTAS2=2"
PSML_DEAL_CTAS=5 run "CTAS=5 CTAS2=2"
run "default again"
timeout 900 python bench.py --task cnn --steps 150 --no-cpu-baseline --no-ring-gemm > gpurun_out/b93c.json 2> gpurun_out/b93c.err
python -c "
import json; d=json.load(open('gpurun_out/b93c.json'))
print('cnn value',round(d['value']),'e2e',round(d['e2e']['value']),'ms',round(d['ms_per_step'],4))"
