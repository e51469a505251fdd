#!/bin/bash
# compute-sanitizer passes over small GPU parity cases (run under gpurun).
TAG=${1:-r01}
mkdir -p gpurun_out
SEL="test_search_config0_bit_exact or test_playouts_edge_cases or test_search_leaf_bit_exact or test_gen_positions or test_playouts_bit_exact or test_playouts_ex_stream_key or test_hosted_hybrid_iteration_mode_bit_exact"
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 --error-exitcode 99 \
    python -m pytest tests/test_gpu_parity.py tests/test_gpu_hosted.py -m gpu -q -x -k "$SEL" > gpurun_out/${TAG}_sanitizer_${tool}.log 2>&1
  echo "$tool rc=$?"; grep -E "ERROR SUMMARY|passed|failed" gpurun_out/${TAG}_sanitizer_${tool}.log | tail -2
done
