#!/bin/bash
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
timeout 600 python bench.py --sweep --sweep-ms 200 > gpurun_out/r07_sweep_fig5.json 2> gpurun_out/r07_sweep.err; echo "sweep rc=$?"
BENCH_BACKEND=gloo BENCH_SAME_DEVICE=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
  --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --steps 10 --warmup 3 --no-cpu \
  > gpurun_out/r07_bench_2rank_gloo.json 2> gpurun_out/r07_bench_2rank.err; echo "2rank rc=$?"
