#!/bin/bash
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
timeout 700 python bench.py --selfplay 16 --h2h --h2h-schemes tree,block --move-ms 500 > gpurun_out/r06_h2h_tree_vs_block.json 2> gpurun_out/r06_h2h_tree.err; echo "h2h rc=$?"
timeout 700 python bench.py --selfplay 16 --sp-scheme tree --move-ms 500 > gpurun_out/r06_selfplay16_tree.json 2> gpurun_out/r06_selfplay_tree.err; echo "sp rc=$?"
