cd $GRAFT_REPO_ROOT
timeout 120 python -m pytest tests/test_gpu_tc.py -q -x -k "ring_gemm_bitexact and 64 and 128-32-64" 2>&1 | tail -3
timeout 600 python -m pytest tests/test_gpu_tc.py tests/test_gpu_split.py tests/test_gpu_tc_fullsize.py -q -x 2>&1 | tail -3
timeout 300 python tools/tc_sweep.py 1024,2048,4096,8192 2>&1 | grep '"backend": 2' | grep '"l": 64'
PSML_TC_V4=1 timeout 300 python tools/tc_sweep.py 4096,8192 2>&1 | grep '"backend": 2' | grep '"l": 64'
