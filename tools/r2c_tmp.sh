mkdir -p gpurun_out
T=${1:-r2d}
for f in test_gpu_hooks test_gpu_runtime test_gpu_parity test_gpu_workloads test_gpu_sharded; do
  timeout 600 python -u -m pytest tests/$f.py -x -q -m gpu --timeout=300 --timeout-method=thread -p no:cacheprovider > gpurun_out/${T}_$f.log 2>&1
  echo "rc=$?" >> gpurun_out/${T}_$f.log
done
timeout 600 python tools/hook_bench.py > gpurun_out/${T}_hook_bench.json 2> gpurun_out/${T}_hook_bench.err
timeout 900 compute-sanitizer --tool synccheck --print-limit 30 python tools/sanitize_driver.py > gpurun_out/${T}_sanitize_synccheck.log 2>&1; echo "rc=$?" >> gpurun_out/${T}_sanitize_synccheck.log
