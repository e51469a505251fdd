#!/bin/bash
# Leaf-parallel kernel shakedown (run under gpurun): one search per process
# under its own timeout, growing grids, iteration and time mode.
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
T=${1:-r2}
for cfg in "128 5" "1024 5" "16384 8" "16384 40" "65536 20" "128 0 30" "16384 0 50" "16384 0 500" "65536 0 200"; do
  timeout 90 python tools/leaf_debug.py $cfg >> gpurun_out/${T}_leafdbg.txt 2>&1; echo "rc=$? $cfg" >> gpurun_out/${T}_leafdbg.txt
done
cat gpurun_out/${T}_leafdbg.txt
