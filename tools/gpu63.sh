cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for t in cnn; do
for c in 4 16 0; do
PSML_DEAL_CTAS=$c timeout 900 python bench.py --task $t --steps 150 --no-cpu-baseline --no-ring-gemm > gpurun_out/b63.json 2> gpurun_out/b63.err
python -c "
import json; d=json.load(open('gpurun_out/b63.json'))
print('$t CTAS=$c value',round(d['value']),'online',round(d['online_samples_per_s']),'ms',round(d['ms_per_step'],4), 'dealer_ms', round(d['kernel_classes']['dealer']['ms_per_step'],4))"
done
done
