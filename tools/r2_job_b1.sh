mkdir -p gpurun_out/golden5/cfg5_parts
cp tests/golden/fullsize/cfg5_parts/*.json gpurun_out/golden5/cfg5_parts/
T=r2n
timeout 600 python -u -m pytest tests/test_gpu_hooks.py tests/test_gpu_workloads.py -x -q -m gpu --timeout=300 --timeout-method=thread -p no:cacheprovider > gpurun_out/${T}_pytest.log 2>&1
echo "rc=$?" >> gpurun_out/${T}_pytest.log
timeout 420 python tools/hook_bench.py --lulesh-steps 30 > gpurun_out/${T}_hook_a.json 2> gpurun_out/${T}_hook_a.err
XPL_WORK_PATH=paper_conf_ipps_pirkelbauerlvl20_b200/libxplwork_ab.so timeout 420 python tools/hook_bench.py --lulesh-steps 30 > gpurun_out/${T}_hook_b.json 2> gpurun_out/${T}_hook_b.err
timeout 2700 python tools/golden_fullsize.py cfg5 --only g0,g1,g2,g3,g4,g5 --workers 6 --no-merge --out gpurun_out/golden5 > gpurun_out/golden5/log_b1.txt 2>&1
echo "rc=$?" >> gpurun_out/golden5/log_b1.txt
