#!/bin/bash
# One gpurun job (replaces the per-run scripts of round 1):
#   gpurun --timeout S -- bash tools/gpu_job.sh TAG STEP [STEP ...]
# Runs the steps in order on the GPU box; every step logs to gpurun_out/TAG_<step>.*
# Steps:
#   build                  make the libraries (they normally travel in-tree)
#   smoke                  __graft_entry__.smoke()
#   pytest[:ARGS]          python -m pytest tests -q -m gpu ARGS  (ARGS: '+'-separated, e.g. -k+lulesh)
#   bench[:ARGS]           python bench.py ARGS > TAG_bench.json
#   launches               ncu launch list (gpu__time_duration.sum) of a short bench run
#   ncu:REGEX[:SKIP[:CMD]] ncu --set full of one launch of kernel REGEX (default command: bench.py --step-only)
#   py:SCRIPT[:ARGS]       python SCRIPT ARGS > TAG_<name>.json
#   pyab:SCRIPT[:ARGS]     the same with the A/B build libxplwork_ab.so > TAG_<name>_ab.json
#   pyw:LIB:SCRIPT[:ARGS]  the same with the work library LIB (an A/B build in the package dir)
#   sanitize:TOOL          compute-sanitizer --tool TOOL (memcheck|synccheck|racecheck) over tools/sanitize_driver.py
#   bench2[:ARGS]          2 ranks on this one GPU over gloo (the sharded N>1 bench path): torchrun bench.py --gpus 2
#   golden5                cfg5's oracle expectations on the box's host cores (tools/golden_fullsize.py cfg5)
#   hookab                 tools/hook_bench.py with libxplwork.so and with the A/B build libxplwork_ab.so
TAG=$1; shift
mkdir -p gpurun_out
echo "nproc=$(nproc) $(nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader)" > gpurun_out/${TAG}_box.txt
for step in "$@"; do
  kind=${step%%:*}; rest=${step#*:}; [ "$rest" = "$step" ] && rest=""
  args=${rest//+/ }
  case $kind in
    build) make -s -C paper_conf_ipps_pirkelbauerlvl20_b200/csrc -j8 > gpurun_out/${TAG}_build.log 2>&1 ;;
    smoke) python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1
           echo "rc=$?" >> gpurun_out/${TAG}_smoke.log ;;
    pytest) timeout 2400 python -u -m pytest tests -q -m gpu --durations=15 --timeout=1200 --timeout-method=thread \
              -p no:cacheprovider $args > gpurun_out/${TAG}_pytest.log 2>&1
            echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest.log ;;
    bench) timeout 1800 python bench.py $args > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err ;;
    launches) timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv \
                --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 1 --warmup 1 --step-only \
                > gpurun_out/${TAG}_launches.log 2>&1 ;;
    ncu) re=${rest%%:*}; r2=${rest#*:}; [ "$r2" = "$rest" ] && r2=""
         skip=${r2%%:*}; cmd=${r2#*:}; [ "$cmd" = "$r2" ] && cmd=""
         [ -z "$skip" ] && skip=0; [ -z "$cmd" ] && cmd="bench.py --step-only --steps 1 --warmup 0"
         name=$(echo "$re" | tr -cd 'A-Za-z0-9_')
         timeout 1200 ncu --set full --import-source on --clock-control none -k "regex:$re" --launch-skip $skip \
           --launch-count 1 -o gpurun_out/${TAG}_ncu_$name python ${cmd//+/ } > gpurun_out/${TAG}_ncu_$name.log 2>&1 ;;
    py) script=${rest%%:*}; a2=${rest#*:}; [ "$a2" = "$rest" ] && a2=""
        name=$(basename "$script" .py)
        timeout 1800 python $script ${a2//+/ } > gpurun_out/${TAG}_$name.json 2> gpurun_out/${TAG}_$name.err ;;
    pyw) lib=${rest%%:*}; r2=${rest#*:}; script=${r2%%:*}; a2=${r2#*:}; [ "$a2" = "$r2" ] && a2=""
         name=$(basename "$script" .py)_$(basename "$lib" .so)
         XPL_WORK_PATH=paper_conf_ipps_pirkelbauerlvl20_b200/$lib timeout 1800 python $script ${a2//+/ } \
           > gpurun_out/${TAG}_$name.json 2> gpurun_out/${TAG}_$name.err ;;
    pyab) script=${rest%%:*}; a2=${rest#*:}; [ "$a2" = "$rest" ] && a2=""
          name=$(basename "$script" .py)
          XPL_WORK_PATH=paper_conf_ipps_pirkelbauerlvl20_b200/libxplwork_ab.so timeout 1800 python $script ${a2//+/ } \
            > gpurun_out/${TAG}_${name}_ab.json 2> gpurun_out/${TAG}_${name}_ab.err ;;
    sanitize) timeout 1500 compute-sanitizer --tool $rest --print-limit 50 python tools/sanitize_driver.py \
                > gpurun_out/${TAG}_sanitize_$rest.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_sanitize_$rest.log ;;
    bench2) XPL_DIST_BACKEND=gloo timeout 1800 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
              --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 $args \
              > gpurun_out/${TAG}_bench2.json 2> gpurun_out/${TAG}_bench2.err ;;
    golden5) mkdir -p gpurun_out/golden5/cfg5_parts
             # (a part peaks near 28 GB of host memory: GOLDEN5_GB (default 40) of MemAvailable per worker)
             W=$(python -c "import os; m=int(open('/proc/meminfo').read().split('MemAvailable:')[1].split()[0])/2**20; print(max(1, min(os.cpu_count()-1, int(m//int(os.environ.get('GOLDEN5_GB', '40'))))))")
             echo "workers=$W" > gpurun_out/golden5/box.txt; free -g >> gpurun_out/golden5/box.txt
             cp tests/golden/fullsize/cfg5_parts/*.json gpurun_out/golden5/cfg5_parts/ 2>/dev/null
             timeout ${GOLDEN5_TIMEOUT:-5400} python tools/golden_fullsize.py cfg5 --workers $W --out gpurun_out/golden5 \
               ${GOLDEN5_ONLY:+--only $GOLDEN5_ONLY --no-merge} > gpurun_out/golden5/log.txt 2>&1
             echo "rc=$?" >> gpurun_out/golden5/log.txt ;;
    hookab) timeout 900 python tools/hook_bench.py --lulesh-steps 30 > gpurun_out/${TAG}_hook_a.json 2> gpurun_out/${TAG}_hook_a.err
            XPL_WORK_PATH=paper_conf_ipps_pirkelbauerlvl20_b200/libxplwork_ab.so timeout 900 python tools/hook_bench.py \
              --lulesh-steps 30 > gpurun_out/${TAG}_hook_b.json 2> gpurun_out/${TAG}_hook_b.err ;;
    *) echo "unknown step $step" >> gpurun_out/${TAG}_box.txt ;;
  esac
done
