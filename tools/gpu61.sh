cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_primitives.py -x -q -k "secure_matmul" 2>&1 | tail -2
timeout 900 python -m pytest tests/test_gpu_training.py -x -q -k "bitexact or graph" 2>&1 | tail -2
for t in linreg logreg cnn; do
timeout 900 python bench.py --task $t --steps 200 --no-cpu-baseline --no-ring-gemm > gpurun_out/b61_$t.json 2> gpurun_out/b61_$t.err
tail -1 gpurun_out/b61_$t.err
python -c "
import json; d=json.load(open('gpurun_out/b61_$t.json'))
print('$t value',round(d['value']),'online',round(d['online_samples_per_s']),'infer',round(d['infer_samples_per_s']),'e2e',round(d['e2e']['value']),'ms',round(d['ms_per_step'],4)); print({k:(round(v['ms_per_step'],4), v['launches_per_step']) for k,v in d['kernel_classes'].items()})"
done
timeout 600 python -c "
import sys; sys.path.insert(0,'.')
import bench
print(bench.beaver_latency_figure())
"
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches61_cnn.csv python tools/step_profile.py cnn 2 > gpurun_out/ncu61.log 2>&1
