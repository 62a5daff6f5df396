mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_um_counters.py -x -q -m gpu -k "page or um_" > gpurun_out/r1w_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r1w_pytest.log
timeout 300 python tools/page_bench.py > gpurun_out/r1w_page.json 2> gpurun_out/r1w_page.err
timeout 600 ncu --set full --import-source on --clock-control none -k regex:page_kernel --launch-skip 1 --launch-count 1 -o gpurun_out/r1w_page python tools/page_bench.py > gpurun_out/r1w_ncu.log 2>&1
