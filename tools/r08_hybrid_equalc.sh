#!/bin/bash
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
timeout 1300 python bench.py --selfplay 32 --sp-scheme hybrid --move-ms 500 > gpurun_out/r08_selfplay32_hybrid_equalC.json 2>/dev/null; echo "hybrid rc=$?"
