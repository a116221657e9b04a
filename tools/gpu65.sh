cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import oracle; oracle.build()"
timeout 1500 python tools/cfg5_sweep.py > gpurun_out/cfg5_sweep.jsonl 2> gpurun_out/cfg5.err
tail -3 gpurun_out/cfg5.err; cat gpurun_out/cfg5_sweep.jsonl
