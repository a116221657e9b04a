cd $GRAFT_REPO_ROOT
timeout 600 python tools/mm_prof.py 2>&1 | tail -12
