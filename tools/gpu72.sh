cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
run() {
  timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-ring-gemm > gpurun_out/b72.json 2> gpurun_out/b72.err
  python -c "
import json; d=json.load(open('gpurun_out/b72.json'))
print('$1 value',round(d['value']),'e2e',round(d['e2e']['value']),'ms',round(d['ms_per_step'],4), d['clocks']['sm_mhz'], 'offline', {k:(round(v,4) if isinstance(v,float) else v) for k,v in d['offline'].items()})" 2>&1 | tail -1
}
run "AFTER=1 default"
for c in 4 6 8 0; do PSML_DEAL_CTAS=$c run "AFTER=1 CTAS=$c"; done
for k in 1 2 8; do PSML_DEAL_KS=$k run "AFTER=1 KS=$k"; done
PSML_SEG=simt run "AFTER=1 SEG=simt"
PSML_DEAL_AFTER=2 PSML_DEAL_CTAS=6 run "AFTER=2 CTAS=6"
PSML_DEAL_AFTER=0 run "AFTER=0"
run "AFTER=1 default again"
