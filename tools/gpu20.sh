cd $GRAFT_REPO_ROOT
timeout 1500 python -m pytest tests -m gpu -q -rA 2>&1 | grep -E "passed|failed|one-epoch|Error" | tail -12
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
