#!/bin/bash
# 32 more equal-C games of the NEXT-1 hybrid (block + host trees) vs the 16-thread CPU oracle, an independent seed set.
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
timeout 1300 python bench.py --selfplay 32 --sp-scheme hybrid --move-ms 500 --sp-seed-base 100000 > gpurun_out/r09_selfplay32_hybrid_equalC_s100k.json 2>gpurun_out/r09_selfplay_hybrid.err; echo "hybrid rc=$?"
