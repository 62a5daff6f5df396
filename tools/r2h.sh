# round-2 GPU job: sanitizers, the N>1 sharded bench path (gloo on one GPU), ncu of the hot kernels
mkdir -p gpurun_out
T=${1:-r2h}
for tool in memcheck racecheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 30 python tools/sanitize_driver.py > gpurun_out/${T}_sanitize_$tool.log 2>&1
  echo "rc=$?" >> gpurun_out/${T}_sanitize_$tool.log
done
XPL_DIST_BACKEND=gloo timeout 1200 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 1 --warmup 1 --timesteps 5 > gpurun_out/${T}_bench_2rank_gloo.json 2> gpurun_out/${T}_bench_2rank_gloo.err
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_integrate_stress --launch-skip 2 --launch-count 1 -o gpurun_out/${T}_ncu_stress python bench.py --step-only --steps 1 --warmup 0 --timesteps 3 > gpurun_out/${T}_ncu_stress.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:fold_kernel --launch-skip 40 --launch-count 1 -o gpurun_out/${T}_ncu_fold python bench.py --step-only --steps 1 --warmup 0 --timesteps 3 > gpurun_out/${T}_ncu_fold.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:diag_tile --launch-skip 2 --launch-count 1 -o gpurun_out/${T}_ncu_diag python bench.py --step-only --steps 1 --warmup 0 --timesteps 3 > gpurun_out/${T}_ncu_diag.log 2>&1
timeout 600 python tools/hook_bench.py > gpurun_out/${T}_hook_bench.json 2> gpurun_out/${T}_hook_bench.err
timeout 1800 python bench.py > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.err
