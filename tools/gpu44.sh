cd $GRAFT_REPO_ROOT
for cfg in "1 1" "1 0" "2 1" "4 1" "0 1"; do
set -- $cfg
PSML_DEAL_CTAS=$1 PSML_PRIO=$2 timeout 300 python bench.py --steps 2000 --no-cpu-baseline --no-ring-gemm > gpurun_out/b44.json 2> gpurun_out/b44.err
python -c "
import json; d=json.load(open('gpurun_out/b44.json'))
print('CTAS=$1 PRIO=$2 value',round(d['value']),'online_graph',round(d.get('online_graph_samples_per_s')),'e2e',round(d['e2e']['value']),'ms',round(d['ms_per_step'],4), 'dealer_eager_ms', round(d['kernel_classes']['dealer']['ms_per_step'],4))"
done
