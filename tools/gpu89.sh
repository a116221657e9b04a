cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python bench.py > gpurun_out/b89.json 2> gpurun_out/b89.err
python -c "
import json; d=json.load(open('gpurun_out/b89.json'))
print('value',round(d['value']),'e2e',round(d['e2e']['value']),'online_graph',round(d['online_graph_samples_per_s']),'ms',round(d['ms_per_step'],4), d['clocks'], d['roofline']['frac'], d['roofline']['traffic'])"
timeout 600 python bench.py --impl reference --steps 20 --warmup 3 2>&1 | tail -1 | cut -c1-400
