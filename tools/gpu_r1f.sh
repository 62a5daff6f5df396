set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r1f_smi.txt 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r1f_smoke.log 2>&1
timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/r1f_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r1f_pytest.log
timeout 900 python bench.py > gpurun_out/r1f_bench.json 2> gpurun_out/r1f_bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file gpurun_out/r1f_launches.csv python bench.py --step-only --steps 2 --warmup 3 > /dev/null 2>&1
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 3000 --csv --log-file gpurun_out/r1f_traffic.csv python bench.py --step-only --steps 2 --warmup 3 > /dev/null 2>&1
ls -la gpurun_out
