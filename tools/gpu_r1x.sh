set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r1x_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/r1x_smoke.log
timeout 1500 python -m pytest tests -x -q -m gpu --durations=5 > gpurun_out/r1x_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r1x_pytest.log
timeout 900 python bench.py > gpurun_out/r1x_bench.json 2> gpurun_out/r1x_bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file gpurun_out/r1x_launches.csv python bench.py --step-only --steps 2 --warmup 3 > /dev/null 2>&1
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 3000 --csv --log-file gpurun_out/r1x_traffic.csv python bench.py --step-only --steps 2 --warmup 3 > /dev/null 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:fold_kernel --launch-skip 400 --launch-count 1 -o gpurun_out/r1x_fold python bench.py --step-only --steps 1 --warmup 3 > gpurun_out/r1x_ncu_fold.log 2>&1
