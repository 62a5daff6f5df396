mkdir -p gpurun_out
T=${1:-r2g}
timeout 1500 python -u -m pytest tests -q -m gpu --timeout=900 --timeout-method=thread -p no:cacheprovider --durations=12 > gpurun_out/${T}_pytest.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_pytest.log
timeout 1500 python bench.py > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.err
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none -c 5000 --csv --log-file gpurun_out/${T}_launches.csv python bench.py --steps 1 --warmup 1 --step-only --timesteps 10 > gpurun_out/${T}_launches.log 2>&1
