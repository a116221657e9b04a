cd $GRAFT_REPO_ROOT
timeout 300 python -m pytest tests/test_gpu_training.py -q -x -k "graph or bitexact" 2>&1 | tail -15
