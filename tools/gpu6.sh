cd $GRAFT_REPO_ROOT
timeout 300 python tools/tc_sweep.py 512,1024,2048,4096,8192 2>&1 | tail -20
timeout 300 ncu --set full --clock-control none --import-source on -k regex:tc_ring_gemm -c 1 -o gpurun_out/tc4096 python tools/tc_sweep.py 4096 > gpurun_out/ncu_tc.log 2>&1
tail -3 gpurun_out/ncu_tc.log
