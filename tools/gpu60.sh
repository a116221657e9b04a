cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_split.py -x -q 2>&1 | tail -3
timeout 900 python bench.py --steps 300 --no-cpu-baseline > gpurun_out/b60.json 2> gpurun_out/b60.err
tail -2 gpurun_out/b60.err
python -c "
import json; d=json.load(open('gpurun_out/b60.json'))
print('value',round(d['value']),'infer',round(d['infer_samples_per_s']),'e2e',round(d['e2e']['value']),'ms',round(d['ms_per_step'],4)); print(d['beaver_matmul_cfg1'])"
