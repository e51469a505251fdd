#!/bin/bash
# Round validation on the GPU box (run under gpurun): GPU tests, smoke, bench,
# reference arm, ncu launch list + --set full captures (tools/profile_round.sh).
# usage: tools/round_validate.sh TAG [pytest -k expr]
TAG=${1:-r2a}; K=${2:-}
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/${TAG}_gpu.txt
if [ -n "$K" ]; then KA=(-k "$K"); else KA=(); fi
timeout 1500 python -m pytest tests -m gpu -q --timeout 300 --timeout_method=thread "${KA[@]}" > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/${TAG}_pytest_gpu.log
timeout 120 python __graft_entry__.py smoke > gpurun_out/${TAG}_smoke.log 2>&1; echo "smoke rc=$?"
timeout 400 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err; echo "bench rc=$?"
timeout 300 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/${TAG}_bench_reference.json 2>&1; echo "ref rc=$?"
tools/profile_round.sh ${TAG}
