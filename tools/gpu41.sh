cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_primitives.py -q -x 2>&1 | tail -30
