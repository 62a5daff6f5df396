set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r1final4_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/r1final4_smoke.log
timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/r1final4_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r1final4_pytest.log
timeout 900 python bench.py > gpurun_out/r1final4_bench.json 2> gpurun_out/r1final4_bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r1final4_launches.csv python bench.py --steps 2 --warmup 1 > gpurun_out/r1final4_ncu_bench.log 2>&1
