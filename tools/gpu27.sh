cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests/test_gpu_split.py -q -x 2>&1 | tail -15
