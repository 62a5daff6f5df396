set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r1final2_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/r1final2_smoke.log
timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/r1final2_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r1final2_pytest.log
timeout 900 python bench.py > gpurun_out/r1final2_bench.json 2> gpurun_out/r1final2_bench.err
