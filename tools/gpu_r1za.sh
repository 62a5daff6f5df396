# A/B: nw's reads through xpl_read_lat (deferred commit, new) vs xpl_read (pre2 = scratch/pre2)
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_workloads.py tests/test_gpu_fullsize.py tests/test_gpu_parity.py -x -q -m gpu -k "nw or read_lat" > gpurun_out/r1za_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r1za_pytest.log
for v in pre2 new pre2 new pre2 new; do
  if [ $v = new ]; then unset XPL_LIB_PATH XPL_WORK_PATH; else export XPL_LIB_PATH=$PWD/scratch/$v/libxpl.so XPL_WORK_PATH=$PWD/scratch/$v/libxplwork.so; fi
  timeout 600 python bench.py --no-cpu-baseline --no-other-configs --steps 5 --warmup 3 > /tmp/b.json 2>/dev/null
  python -c "import json;d=json.load(open('/tmp/b.json'));l=d['launch_log'];print('$v', round(d['value']/1e9,4), round(d['ms_per_step'],3), round(l['nw_kernel_upper']['epoch_ms_sum']+l['nw_kernel_lower']['epoch_ms_sum'],3), round(d['breakdown_ms_per_step']['instrumented_kernels'],3))" >> gpurun_out/r1za_ab.txt
done
