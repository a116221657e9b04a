cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/t45.txt
cat gpurun_out/t45.txt
timeout 600 python bench.py > gpurun_out/b45.json 2> gpurun_out/b45.err
tail -3 gpurun_out/b45.err
cat gpurun_out/b45.json | head -c 3000
