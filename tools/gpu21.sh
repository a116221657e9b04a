cd $GRAFT_REPO_ROOT
timeout 120 python -m pytest tests/test_gpu_tc.py -q -x -k "ring_gemm_bitexact and 64 and 128-32-64" 2>&1 | tail -4
timeout 300 python -m pytest tests/test_gpu_tc.py tests/test_gpu_split.py -q -x 2>&1 | tail -4
timeout 300 python tools/tc_sweep.py 2048,4096,8192 2>&1 | grep '"backend": 2' | tail -12
