set -x
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -x -q -m gpu --durations=10 > gpurun_out/r1n_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r1n_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r1n_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/r1n_smoke.log
timeout 300 python tools/um_faults.py > gpurun_out/r1n_um.json 2> gpurun_out/r1n_um.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 4000 --csv --log-file gpurun_out/r1n_launches.csv python bench.py --step-only --steps 2 --warmup 1 > gpurun_out/r1n_ncu_launch.log 2>&1
timeout 900 python bench.py > gpurun_out/r1n_bench.json 2> gpurun_out/r1n_bench.err
