#!/bin/bash
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
timeout 1300 python bench.py --selfplay 32 --move-ms 500 > gpurun_out/r08_selfplay32_block_equalC.json 2>/dev/null; echo "block rc=$?"
timeout 1300 python bench.py --selfplay 32 --sp-scheme tree --move-ms 500 > gpurun_out/r08_selfplay32_tree_equalC.json 2>/dev/null; echo "tree rc=$?"
