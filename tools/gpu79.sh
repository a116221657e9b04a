cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for c in 4 8 16 0; do
PSML_DEAL_CTAS=$c timeout 900 python bench.py --task cnn --steps 150 --no-cpu-baseline --no-ring-gemm > gpurun_out/b79c.json 2> gpurun_out/b79c.err
python -c "
import json; d=json.load(open('gpurun_out/b79c.json'))
print('cnn CTAS=$c value',round(d['value']),'e2e',round(d['e2e']['value']),'ms',round(d['ms_per_step'],4), 'offline', round(d['offline']['ms_per_step'],4))"
done
timeout 300 python tools/timeline.py cnn 6 gpurun_out/timeline_cnn2.json 2>&1 | grep -E "mean step|busy|deal_prg|ring_gemm_small"
