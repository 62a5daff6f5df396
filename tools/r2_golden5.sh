# cfg5's oracle expectations on the GPU box's host cores (CPU only: 16 cores, large RAM);
# the parts land in gpurun_out/golden5/cfg5_parts/, the merged file in gpurun_out/golden5/cfg5.json
mkdir -p gpurun_out/golden5
W=$(python -c "import os; m=os.sysconf('SC_PAGE_SIZE')*os.sysconf('SC_PHYS_PAGES')/2**30; print(max(1, min(os.cpu_count()-1, int(m//36))))")
echo "workers=$W $(nproc) cores" > gpurun_out/golden5/box.txt; free -g >> gpurun_out/golden5/box.txt
python tools/golden_fullsize.py cfg5 --workers $W --out gpurun_out/golden5 > gpurun_out/golden5/log.txt 2>&1
echo "rc=$?" >> gpurun_out/golden5/log.txt
