#!/bin/bash
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
timeout 1200 python bench.py --selfplay 32 --sp-scheme tree --move-ms 500 > gpurun_out/r07_selfplay32_tree.json 2>/dev/null; echo "tree rc=$?"
timeout 1200 python bench.py --selfplay 32 --h2h --h2h-schemes tree,block --move-ms 500 > gpurun_out/r07_h2h32_tree_vs_block.json 2>/dev/null; echo "h2h rc=$?"
