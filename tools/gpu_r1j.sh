set -x
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -x -q -m gpu --durations=8 > gpurun_out/r1j_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r1j_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r1j_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/r1j_smoke.log
timeout 900 python bench.py > gpurun_out/r1j_bench.json 2> gpurun_out/r1j_bench.err
