#!/bin/bash
# Depth statistic: GPU suite, then Fig. 8 analog games (mean tree depth per game step).
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/r07c_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/r07c_pytest_gpu.log
[ -n "$SKIP_GAMES" ] && exit 0
timeout 300 python bench.py --no-cpu --steps 10 > gpurun_out/r07c_bench.json 2>/dev/null; echo "bench rc=$?"
timeout 700 python bench.py --selfplay 8 --move-ms 500 > gpurun_out/r07_fig8_block.json 2>/dev/null; echo "block rc=$?"
timeout 700 python bench.py --selfplay 8 --move-ms 500 --sp-scheme hybrid > gpurun_out/r07_fig8_hybrid.json 2>/dev/null; echo "hybrid rc=$?"
timeout 700 python bench.py --selfplay 8 --move-ms 500 --sp-scheme tree > gpurun_out/r07_fig8_tree.json 2>/dev/null; echo "tree rc=$?"
