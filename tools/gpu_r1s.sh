mkdir -p gpurun_out
for v in prof noprof prof noprof; do
  if [ $v = noprof ]; then export XPL_BENCH_NOPROF=1; else unset XPL_BENCH_NOPROF; fi
  timeout 600 python bench.py --no-cpu-baseline --no-other-configs --steps 5 --warmup 3 > /tmp/b.json 2>/tmp/b.err
  python -c "import json;d=json.load(open('/tmp/b.json'));print('$v', round(d['value']/1e9,4), round(d['ms_per_step'],3), round(d['e2e']['value']/1e9,4))" >> gpurun_out/r1s_prof.txt 2>&1 || tail -3 /tmp/b.err >> gpurun_out/r1s_prof.txt
done
