mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_launch_log.py -x -q -m gpu -k "page or launch" > gpurun_out/r1p_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r1p_pytest.log
for v in base f4 base f4; do
  if [ $v = base ]; then unset XPL_LIB_PATH XPL_WORK_PATH; else export XPL_LIB_PATH=$PWD/scratch/$v/libxpl.so XPL_WORK_PATH=$PWD/scratch/$v/libxplwork.so; fi
  timeout 600 python bench.py --no-cpu-baseline --no-other-configs --steps 5 --warmup 3 > /tmp/b.json 2>/dev/null
  python -c "import json;d=json.load(open('/tmp/b.json'));print('$v', round(d['value']/1e9,4), round(d['ms_per_step'],3), json.dumps(d['runtime_kernels']['fold']), json.dumps(d['diagnose_at_scale']['record']['fold_gbs']), json.dumps(d['diagnose_at_scale'].get('page_view')))" >> gpurun_out/r1p_step.txt
done
