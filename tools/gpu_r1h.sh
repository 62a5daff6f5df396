# A/B of diagnose staging depth / occupancy variants (scratch/vN builds)
mkdir -p gpurun_out
for v in v0 v1 v2 v3 v4; do
  if [ $v = v0 ]; then unset XPL_LIB_PATH XPL_WORK_PATH; else export XPL_LIB_PATH=$PWD/scratch/$v/libxpl.so XPL_WORK_PATH=$PWD/scratch/$v/libxplwork.so; fi
  for r in 1 2; do echo "$v $(timeout 300 python tools/diag_bench.py)" >> gpurun_out/r1h_diag.txt; done
  echo "$v $(timeout 400 python bench.py --no-cpu-baseline --no-other-configs --steps 5 --warmup 3)" >> gpurun_out/r1h_step.txt
done
