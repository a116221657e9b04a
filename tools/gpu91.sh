cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python bench.py --task cnn --steps 200 --no-ring-gemm --no-cpu-baseline > gpurun_out/r01d_bench_cnn.json 2> gpurun_out/b91c.err
python -c "
import json; d=json.load(open('gpurun_out/r01d_bench_cnn.json'))
print('cnn value',round(d['value']),'e2e',round(d['e2e']['value']),'online',round(d['online_samples_per_s']),'ms',round(d['ms_per_step'],4), d['clocks'])"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"conv_gw_image|msb_chain" -c 3 -f -o gpurun_out/r01d_cnn python tools/step_profile.py cnn 1 > gpurun_out/ncu91.log 2>&1; echo "ncu rc=$?"; tail -2 gpurun_out/ncu91.log
timeout 300 python tools/timeline.py mlp 20 gpurun_out/timeline_final.json 2>&1 | tail -45
