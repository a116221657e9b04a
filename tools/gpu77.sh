cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_training.py -x -q -k "step_host or graph_replay" 2>&1 | tail -2
timeout 900 python bench.py --no-cpu-baseline --no-ring-gemm > gpurun_out/b77.json 2> gpurun_out/b77.err
python -c "
import json; d=json.load(open('gpurun_out/b77.json'))
print('value',round(d['value']),'e2e',d['e2e'],'online_graph',round(d['online_graph_samples_per_s']),'ms',round(d['ms_per_step'],4), d['clocks'])"
timeout 900 python bench.py --task cnn --steps 200 --no-cpu-baseline --no-ring-gemm > gpurun_out/b77c.json 2> gpurun_out/b77c.err
python -c "
import json; d=json.load(open('gpurun_out/b77c.json'))
print('cnn value',round(d['value']),'e2e',round(d['e2e']['value']),'online',round(d['online_samples_per_s']),'infer',round(d['infer_samples_per_s']),'ms',round(d['ms_per_step'],4)); print({k:(round(v['ms_per_step'],4), v['launches_per_step']) for k,v in d['kernel_classes'].items()})"
timeout 300 python tools/timeline.py cnn 6 gpurun_out/timeline_cnn.json 2>&1 | tail -40
