mkdir -p gpurun_out
timeout 900 python bench.py > gpurun_out/r1t_bench.json 2> gpurun_out/r1t_bench.err
timeout 600 python -m pytest tests/test_gpu_launch_log.py -x -q -m gpu > gpurun_out/r1t_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r1t_pytest.log
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/r1t_ref.json 2> gpurun_out/r1t_ref.err
