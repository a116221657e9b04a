cd $GRAFT_REPO_ROOT
timeout 120 python -m pytest tests/test_gpu_tc.py -q -x -k "test_tc_ring_gemm_bitexact and 64 and 128-32-64" 2>&1 | tail -15
timeout 300 python -m pytest tests/test_gpu_tc.py -q 2>&1 | tail -25
