cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_training.py -x -q 2>&1 | tail -2
run() {
  timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-ring-gemm > gpurun_out/b69.json 2> gpurun_out/b69.err
  python -c "
import json; d=json.load(open('gpurun_out/b69.json'))
print('$1 value',round(d['value']),'online_graph',round(d.get('online_graph_samples_per_s')),'ms',round(d['ms_per_step'],4),'dealer_ms',round(d['kernel_classes']['dealer']['ms_per_step'],4), d['clocks']['sm_mhz'])"
}
for c in 2 4 6 8; do PSML_DEAL_CTAS=$c run "MINB5 CTAS=$c"; done
PSML_NVCC_EXTRA=-DPSML_DEAL_MINB=6 python -m paper_conf_icpp_chenzzzz020_b200.build --force > /dev/null 2>&1
for c in 4 6 8; do PSML_DEAL_CTAS=$c run "MINB6 CTAS=$c"; done
PSML_NVCC_EXTRA=-DPSML_DEAL_MINB=4 python -m paper_conf_icpp_chenzzzz020_b200.build --force > /dev/null 2>&1
for c in 4; do PSML_DEAL_CTAS=$c run "MINB4 CTAS=$c"; done
