#!/bin/bash
# compute-sanitizer passes over the MCTS_TREE tests (run under gpurun).
TAG=${1:-r06}
mkdir -p gpurun_out
SEL="single_worker_bit_exact or terminal or many_workers_invariants and 148"
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 --error-exitcode 99 \
    python -m pytest tests/test_gpu_tree.py -m gpu -q -x -k "$SEL" > gpurun_out/${TAG}_sanitizer_tree_${tool}.log 2>&1
  echo "$tool rc=$?"; grep -E "ERROR SUMMARY|passed|failed" gpurun_out/${TAG}_sanitizer_tree_${tool}.log | tail -2
done
