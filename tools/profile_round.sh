#!/bin/bash
# Round profile (run under gpurun): ncu launch list of a short bench run plus
# one --set full capture of the playout and block-search kernels.
# usage: tools/profile_round.sh TAG
TAG=${1:-r01}
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 5 --warmup 3 --no-cpu --search-ms 100 \
  > gpurun_out/${TAG}_launches_bench.log 2>&1; echo "launch list rc=$?"
timeout 400 ncu --set full --clock-control none --import-source on -k regex:playouts_kernel -s 3 -c 1 \
  -o gpurun_out/${TAG}_playouts python bench.py --steps 2 --warmup 3 --no-search --no-cpu > /dev/null 2>&1; echo "ncu playouts rc=$?"
timeout 400 ncu --set full --clock-control none --import-source on -k regex:block_search_kernel -s 1 -c 1 \
  -o gpurun_out/${TAG}_block_search python bench.py --steps 1 --warmup 3 --no-cpu --search-iters 200 > /dev/null 2>&1; echo "ncu search rc=$?"
timeout 400 ncu --set full --clock-control none --import-source on -k regex:leaf_search_kernel -s 1 -c 1 \
  -o gpurun_out/${TAG}_leaf_search python bench.py --steps 1 --warmup 3 --no-cpu --search-iters 200 > /dev/null 2>&1; echo "ncu leaf rc=$?"
timeout 400 ncu --set full --clock-control none --import-source on -k regex:tree_search_kernel -s 1 -c 1 \
  -o gpurun_out/${TAG}_tree_search python bench.py --steps 1 --warmup 3 --no-cpu --search-iters 200 > /dev/null 2>&1; echo "ncu tree rc=$?"
