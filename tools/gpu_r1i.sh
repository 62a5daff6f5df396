set -x
mkdir -p gpurun_out
timeout 900 ncu --set full --import-source on --clock-control none -k regex:diag_tile --launch-skip 23 --launch-count 1 -o gpurun_out/r1i_diag_bfs python bench.py --step-only --steps 1 --warmup 0 > gpurun_out/r1i_ncu1.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:diag_tile --launch-count 1 -o gpurun_out/r1i_diag_scale python tools/diag_bench.py > gpurun_out/r1i_ncu2.log 2>&1
timeout 600 ncu --set full --clock-control none -k regex:touch_kernel --launch-count 1 -o gpurun_out/r1i_touch python tools/diag_bench.py > gpurun_out/r1i_ncu3.log 2>&1
timeout 900 python -m pytest tests/test_gpu_cfg5.py -x -q -m gpu --durations=3 > gpurun_out/r1i_cfg5.log 2>&1; echo "rc=$?" >> gpurun_out/r1i_cfg5.log
timeout 900 python bench.py > gpurun_out/r1i_bench.json 2> gpurun_out/r1i_bench.err
