# A/B: every Rodinia read through xpl_read_lat (new) vs nw's only (pre3 = scratch/pre3)
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_workloads.py tests/test_gpu_fullsize.py -x -q -m gpu > gpurun_out/r1zb_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r1zb_pytest.log
for v in pre3 new pre3 new pre3 new; do
  if [ $v = new ]; then unset XPL_LIB_PATH XPL_WORK_PATH; else export XPL_LIB_PATH=$PWD/scratch/$v/libxpl.so XPL_WORK_PATH=$PWD/scratch/$v/libxplwork.so; fi
  timeout 600 python bench.py --no-cpu-baseline --no-other-configs --steps 5 --warmup 3 > /tmp/b.json 2>/dev/null
  python -c "import json;d=json.load(open('/tmp/b.json'));l=d['launch_log'];print('$v', round(d['value']/1e9,4), round(d['ms_per_step'],3), {k: round(v['epoch_ms_sum'],3) for k,v in l.items()}, round(d['breakdown_ms_per_step']['instrumented_kernels'],3))" >> gpurun_out/r1zb_ab.txt
done
