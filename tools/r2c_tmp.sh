mkdir -p gpurun_out
T=${1:-r2e}
shift
for f in "$@"; do
  timeout 900 python -u -m pytest tests/$f.py -x -q -m gpu --timeout=600 --timeout-method=thread -p no:cacheprovider > gpurun_out/${T}_$f.log 2>&1
  echo "rc=$?" >> gpurun_out/${T}_$f.log
done
timeout 600 python tools/hook_bench.py > gpurun_out/${T}_hook_bench.json 2> gpurun_out/${T}_hook_bench.err
timeout 900 ncu --set full --import-source on --clock-control none -k regex:stream_kernel --launch-skip 5 --launch-count 1 -o gpurun_out/${T}_ncu_stream python tools/hook_bench.py --lulesh-steps 0 --reps 5 > gpurun_out/${T}_ncu_stream.log 2>&1
