cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_training.py -x -q -s -k "bench_path" 2>&1 | grep -E "bench path|passed|failed|Error" | head
