cd $GRAFT_REPO_ROOT/tools/micro && ./gemm_micro
