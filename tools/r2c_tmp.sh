mkdir -p gpurun_out
T=${1:-r2k}
timeout 1200 python -u -m pytest tests/test_gpu_fullsize_cfg34.py tests/test_gpu_runtime.py tests/test_gpu_workloads.py -x -q -m gpu --timeout=1100 --timeout-method=thread -p no:cacheprovider --durations=5 > gpurun_out/${T}_pytest.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_pytest.log
timeout 1200 compute-sanitizer --tool racecheck --print-limit 30 python tools/sanitize_driver.py > gpurun_out/${T}_sanitize_racecheck.log 2>&1; echo "rc=$?" >> gpurun_out/${T}_sanitize_racecheck.log
XPL_DIST_BACKEND=gloo timeout 1200 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 1 --warmup 1 --timesteps 5 > gpurun_out/${T}_bench_2rank_gloo.json 2> gpurun_out/${T}_bench_2rank_gloo.err
timeout 1800 python bench.py > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.err
