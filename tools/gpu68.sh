cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
( time timeout 2400 python -m pytest tests -m gpu -x -q ) > gpurun_out/t68.log 2>&1; tail -3 gpurun_out/t68.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 900 python bench.py > gpurun_out/b68.json 2> gpurun_out/b68.err; tail -c 3000 gpurun_out/b68.json
