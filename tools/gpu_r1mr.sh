mkdir -p gpurun_out
XPL_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 3 --warmup 3 --no-cpu-baseline --no-other-configs > gpurun_out/r1mr_bench.json 2> gpurun_out/r1mr_bench.err; echo "rc=$?" >> gpurun_out/r1mr_bench.err
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/r1mr_ref.json 2> gpurun_out/r1mr_ref.err
