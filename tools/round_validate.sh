#!/bin/bash
# Full round validation on the GPU box: GPU tests, smoke, bench, profiles, self-play.
TAG=${1:-r01}; GAMES=${2:-10}; MS=${3:-500}
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/${TAG}_pytest_gpu.log
timeout 120 python __graft_entry__.py smoke > gpurun_out/${TAG}_smoke.log 2>&1; echo "smoke rc=$?"
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/${TAG}_gpu.txt
timeout 300 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err; echo "bench rc=$?"
timeout 300 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/${TAG}_bench_reference.json 2>&1; echo "ref rc=$?"
tools/profile_round.sh ${TAG}
BENCH_DEBUG=1 timeout 1800 python bench.py --selfplay ${GAMES} --move-ms ${MS} > gpurun_out/${TAG}_selfplay_block.json 2> gpurun_out/${TAG}_selfplay_block.err; echo "selfplay rc=$?"
BENCH_DEBUG=1 timeout 1200 python bench.py --selfplay $(( GAMES / 2 )) --move-ms ${MS} --sp-scheme leaf > gpurun_out/${TAG}_selfplay_leaf.json 2> gpurun_out/${TAG}_selfplay_leaf.err; echo "selfplay leaf rc=$?"
