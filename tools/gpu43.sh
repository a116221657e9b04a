cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_training.py -q -x -k "graph" 2>&1 | tail -2
for pr in 1 0; do
PSML_PRIO=$pr timeout 300 python bench.py --steps 2000 --no-cpu-baseline --no-ring-gemm > gpurun_out/b43.json 2> gpurun_out/b43.err
tail -1 gpurun_out/b43.err
python -c "
import json; d=json.load(open('gpurun_out/b43.json'))
print('PRIO=$pr value',d['value'],'online_graph',d.get('online_graph_samples_per_s'),'e2e',d['e2e']['value'],'ms',d['ms_per_step'])"
done
