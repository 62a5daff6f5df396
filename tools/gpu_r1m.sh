set -x
mkdir -p gpurun_out
timeout 300 python tools/um_faults.py > gpurun_out/r1m_um.json 2> gpurun_out/r1m_um.err
timeout 600 python -m pytest tests/test_gpu_um_counters.py -x -q -m gpu > gpurun_out/r1m_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r1m_pytest.log
