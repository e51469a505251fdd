#!/bin/bash
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
timeout 900 python bench.py --selfplay 6 --fig7 --sp-scheme tree --move-ms 100 > gpurun_out/r07_fig7_tree.json 2>/dev/null; echo "fig7 rc=$?"
timeout 1500 python bench.py --sweep --sweep-ms 200 --sweep-games 4 --move-ms 100 > gpurun_out/r07_sweep_fig5_fig6.json 2>/dev/null; echo "sweep rc=$?"
