set -x
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/r1gridfold_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r1gridfold_pytest.log
timeout 900 python bench.py > gpurun_out/r1gridfold_bench.json 2> gpurun_out/r1gridfold_bench.err
