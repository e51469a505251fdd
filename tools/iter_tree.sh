#!/bin/bash
# MCTS_TREE iteration: tree tests + a bench line with the tree_search leg.
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_tree.py -x -q 2>&1 | tail -15
timeout 300 python bench.py --no-cpu --steps 10 > gpurun_out/bench_tree.json 2> gpurun_out/bench_tree.err; echo "bench rc=$?"
python -c "import json; d=json.load(open('gpurun_out/bench_tree.json')); print('value', d['value']); print('search', d['search']); print('tree', d['tree_search'])"
tail -3 gpurun_out/bench_tree.err
