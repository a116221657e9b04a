cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
PSML_DEAL_AFTER=2 timeout 600 python -m pytest tests/test_gpu_training.py -x -q -k graph 2>&1 | tail -1
run() {
  timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-ring-gemm > gpurun_out/b71.json 2> gpurun_out/b71.err
  python -c "
import json; d=json.load(open('gpurun_out/b71.json'))
print('$1 value',round(d['value']),'e2e',round(d['e2e']['value']),'online_graph',round(d.get('online_graph_samples_per_s')),'ms',round(d['ms_per_step'],4), d['clocks']['sm_mhz'])"
}
for a in 0 1 2 3 4 6 9; do PSML_DEAL_AFTER=$a run "AFTER=$a"; done
for a in 2 3; do for c in 2 6 0; do PSML_DEAL_CTAS=$c PSML_DEAL_AFTER=$a run "AFTER=$a CTAS=$c"; done; done
PSML_DEAL_AFTER=2 timeout 300 python tools/timeline.py mlp 20 gpurun_out/timeline_mlp2.json 2>&1 | tail -44
