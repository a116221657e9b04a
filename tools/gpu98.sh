cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
( timeout 2400 python -m pytest tests -m gpu -x -q ) > gpurun_out/t98.log 2>&1; tail -2 gpurun_out/t98.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 900 python bench.py > gpurun_out/b98.json 2> gpurun_out/b98.err
python -c "
import json; d=json.load(open('gpurun_out/b98.json'))
print('value',round(d['value']),'e2e',round(d['e2e']['value']),'online_graph',round(d['online_graph_samples_per_s']),'ms',round(d['ms_per_step'],4), d['clocks'])"
