mkdir -p gpurun_out
T=${1:-r2i}
shift
for f in "$@"; do
  timeout 1200 python -u -m pytest tests/$f.py -x -q -m gpu --timeout=900 --timeout-method=thread -p no:cacheprovider > gpurun_out/${T}_$f.log 2>&1
  echo "rc=$?" >> gpurun_out/${T}_$f.log
done
timeout 600 python tools/hook_bench.py > gpurun_out/${T}_hook_bench.json 2> gpurun_out/${T}_hook_bench.err
timeout 1500 python bench.py --no-other-configs --no-cpu-baseline > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.err
