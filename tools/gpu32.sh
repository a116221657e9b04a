cd $GRAFT_REPO_ROOT
timeout 600 python bench.py --no-cpu-baseline --no-ring-gemm > gpurun_out/bench12.json 2> gpurun_out/bench12.err
tail -2 gpurun_out/bench12.err
python -c "
import json; d=json.load(open('gpurun_out/bench12.json'))
print('value',round(d['value']),'online_graph',round(d['online_graph_samples_per_s']),'online_eager',round(d['online_samples_per_s']),'e2e',round(d['e2e']['value']),'ms',round(d['ms_per_step'],4))"
