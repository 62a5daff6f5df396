mkdir -p gpurun_out
for f in test_gpu_hooks test_gpu_parity test_gpu_runtime test_gpu_workloads test_gpu_sharded; do
  timeout 420 python -u -m pytest tests/$f.py -x -q -m gpu --timeout=150 --timeout-method=thread -p no:cacheprovider > gpurun_out/r2c_$f.log 2>&1
  echo "rc=$?" >> gpurun_out/r2c_$f.log
done
