set -x
mkdir -p gpurun_out
free -g > gpurun_out/r1g_free.txt; nproc >> gpurun_out/r1g_free.txt
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_workloads.py -x -q -m gpu -k "split or smith" > gpurun_out/r1g_split.log 2>&1; echo "rc=$?" >> gpurun_out/r1g_split.log
timeout 1200 python -m pytest tests/test_gpu_cfg5.py -x -q -m gpu --durations=5 > gpurun_out/r1g_cfg5.log 2>&1; echo "rc=$?" >> gpurun_out/r1g_cfg5.log
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/r1g_bench.json 2> gpurun_out/r1g_bench.err
