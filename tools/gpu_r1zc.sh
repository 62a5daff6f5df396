# A/B: Smith-Waterman cells through xpl_read_lat / xpl_write_lat (new) vs xpl_read / xpl_write (pre4)
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_workloads.py tests/test_gpu_parity.py -x -q -m gpu -k "sw or split or read_lat" > gpurun_out/r1zc_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r1zc_pytest.log
for v in pre4 new pre4 new; do
  if [ $v = new ]; then unset XPL_LIB_PATH XPL_WORK_PATH; else export XPL_LIB_PATH=$PWD/scratch/$v/libxpl.so XPL_WORK_PATH=$PWD/scratch/$v/libxplwork.so; fi
  echo "$v $(timeout 600 python tools/sw_bench.py 2>/dev/null)" >> gpurun_out/r1zc_ab.txt
done
