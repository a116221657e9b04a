cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 4000 --csv --log-file gpurun_out/r01e_launches_bench.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-ring-gemm > gpurun_out/b95_ncu.log 2>&1; echo "launch list rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"seg_gemm|tc_seg|msb_chain|had_fused|deal_prg|ring_gemm_cl|open_list|update_all" -s 16 -c 16 -f -o gpurun_out/r01e_full python tools/step_profile.py mlp 3 > gpurun_out/ncu95.log 2>&1; echo "ncu full rc=$?"; tail -1 gpurun_out/ncu95.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"conv_gw_image" -c 1 -f -o gpurun_out/r01e_conv_gw python tools/step_profile.py cnn 1 > gpurun_out/ncu95c.log 2>&1; echo "ncu conv rc=$?"; tail -1 gpurun_out/ncu95c.log
