cd $GRAFT_REPO_ROOT
timeout 120 python -m pytest tests/test_gpu_tc.py -q -x -k "ring_gemm_bitexact and 64 and 128-32-64" 2>&1 | tail -5
timeout 300 python -m pytest tests/test_gpu_tc.py -q 2>&1 | tail -8
timeout 300 python tools/tc_sweep.py 1024,2048,4096,8192 2>&1 | grep '"backend": 2' | tail -12
timeout 300 ncu --set full --clock-control none --import-source on -k regex:tc_ring_gemm -c 1 -o gpurun_out/tc4096v2 python tools/tc_sweep.py 4096 > gpurun_out/ncu_tc2.log 2>&1
tail -2 gpurun_out/ncu_tc2.log
