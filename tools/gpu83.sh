cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.max.sm --format=csv,noheader
( timeout 2400 python -m pytest tests -m gpu -x -q ) > gpurun_out/t83.log 2>&1; tail -2 gpurun_out/t83.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 900 python bench.py > gpurun_out/b83.json 2> gpurun_out/b83.err
python -c "
import json; d=json.load(open('gpurun_out/b83.json'))
print('value',round(d['value']),'e2e',round(d['e2e']['value']),'online_graph',round(d['online_graph_samples_per_s']),'ms',round(d['ms_per_step'],4), d['clocks'], d['roofline'])"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 4000 --csv --log-file gpurun_out/r01d_launches_bench.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-ring-gemm > gpurun_out/b83_ncu.log 2>&1; echo "launch list rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"seg_gemm|tc_seg|msb_chain|had_fused|deal_prg|ring_gemm_cl|open_list|update_all" -s 16 -c 16 -f -o gpurun_out/r01d_full python tools/step_profile.py mlp 3 > gpurun_out/ncu83.log 2>&1; echo "ncu full rc=$?"; tail -3 gpurun_out/ncu83.log
