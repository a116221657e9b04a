cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_training.py -x -q -k "step_host or graph_replay or bitexact" 2>&1 | tail -2
python - <<'PY'
import torch, ctypes
t = torch.empty(100, dtype=torch.uint8).pin_memory()
cudart = ctypes.CDLL("libcudart.so") if False else None
print("pinned tensor ptr", hex(t.data_ptr()))
PY
timeout 900 python bench.py --no-cpu-baseline --no-ring-gemm > gpurun_out/b78.json 2> gpurun_out/b78.err
python -c "
import json; d=json.load(open('gpurun_out/b78.json'))
print('value',round(d['value']),'e2e',round(d['e2e']['value']),'online_graph',round(d['online_graph_samples_per_s']),'ms',round(d['ms_per_step'],4), d['clocks']['sm_mhz'])"
timeout 900 python bench.py --task cnn --steps 200 --no-cpu-baseline --no-ring-gemm > gpurun_out/b78c.json 2> gpurun_out/b78c.err
python -c "
import json; d=json.load(open('gpurun_out/b78c.json'))
print('cnn value',round(d['value']),'e2e',round(d['e2e']['value']),'online',round(d['online_samples_per_s']),'infer',round(d['infer_samples_per_s']),'ms',round(d['ms_per_step'],4), 'offline', round(d['offline']['ms_per_step'],4))"
PSML_DEAL_AFTER=0 timeout 900 python bench.py --task cnn --steps 200 --no-cpu-baseline --no-ring-gemm > gpurun_out/b78c.json 2> gpurun_out/b78c.err
python -c "
import json; d=json.load(open('gpurun_out/b78c.json'))
print('cnn AFTER=0 value',round(d['value']),'e2e',round(d['e2e']['value']),'ms',round(d['ms_per_step'],4))"
