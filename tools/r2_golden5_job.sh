mkdir -p gpurun_out
T=r2l
timeout 900 python -u -m pytest tests/test_gpu_parity.py tests/test_gpu_workloads.py tests/test_gpu_hooks.py -x -q -m gpu --timeout=600 --timeout-method=thread -p no:cacheprovider > gpurun_out/${T}_pytest.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_pytest.log
XPL_DIST_BACKEND=gloo timeout 1200 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 1 --warmup 1 --timesteps 5 > gpurun_out/${T}_bench_2rank_gloo.json 2> gpurun_out/${T}_bench_2rank_gloo.err
bash tools/r2_golden5.sh
