cd $GRAFT_REPO_ROOT
timeout 300 python tools/mm_shapes.py 2>&1 | tail -20
