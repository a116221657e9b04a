cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_tc_fullsize.py tests/test_gpu_training.py -q -x -k "fullsize or cnn_one_epoch or explicit_mask" -s 2>&1 | grep -E "passed|failed|cnn:|Error|assert" | tail -8
PSML_DIST_BACKEND=gloo PSML_SHARE_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 30 --warmup 3 > gpurun_out/bench_dp2.json 2> gpurun_out/bench_dp2.err
tail -3 gpurun_out/bench_dp2.err; head -c 600 gpurun_out/bench_dp2.json; echo
