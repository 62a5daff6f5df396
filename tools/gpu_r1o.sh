# A/B of the fold grid cap (scratch/fN builds, -DXPL_FOLD_CTAS=148/296/1184; base = 592)
mkdir -p gpurun_out
for v in base f1 f2 f3 base; do
  if [ $v = base ]; then unset XPL_LIB_PATH XPL_WORK_PATH; else export XPL_LIB_PATH=$PWD/scratch/$v/libxpl.so XPL_WORK_PATH=$PWD/scratch/$v/libxplwork.so; fi
  echo "$v $(timeout 300 python tools/epoch_bench.py 3000)" >> gpurun_out/r1o_epoch.txt
  timeout 600 python bench.py --no-cpu-baseline --no-other-configs --steps 5 --warmup 3 > /tmp/b.json 2>/dev/null
  python -c "import json;d=json.load(open('/tmp/b.json'));print('$v', round(d['value']/1e9,4), round(d['ms_per_step'],3), json.dumps(d['runtime_kernels']['fold']), json.dumps(d['diagnose_at_scale']['record']['fold_gbs']), json.dumps(d['diagnose_at_scale'].get('page_view')))" >> gpurun_out/r1o_step.txt
done
