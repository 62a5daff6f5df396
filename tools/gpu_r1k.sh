set -x
mkdir -p gpurun_out
timeout 300 python tools/um_faults.py > gpurun_out/r1k_um.json 2> gpurun_out/r1k_um.err
timeout 900 python -m pytest tests/test_gpu_launch_log.py tests/test_gpu_um_counters.py tests/test_gpu_parity.py -x -q -m gpu -k "launch or um_ or page" > gpurun_out/r1k_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r1k_pytest.log
