#!/bin/bash
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
timeout 900 python bench.py --selfplay 6 --fig7 --move-ms 100 > gpurun_out/r08_fig7_block_equalC.json 2>/dev/null; echo "block rc=$?"
timeout 900 python bench.py --selfplay 6 --fig7 --sp-scheme tree --move-ms 100 > gpurun_out/r08_fig7_tree_equalC.json 2>/dev/null; echo "tree rc=$?"
