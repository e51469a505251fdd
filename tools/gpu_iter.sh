#!/bin/bash
# One build->measure iteration on the GPU box (run under gpurun).
# usage: tools/gpu_iter.sh TAG [pytest -k expr]
TAG=${1:-iter}; K=${2:-playouts}
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -x -q -k "$K" 2>&1 | tail -2
timeout 300 python bench.py --no-cpu --steps 20 > gpurun_out/bench_$TAG.log 2> gpurun_out/bench_$TAG.err; echo "bench rc=$?"
cat gpurun_out/bench_$TAG.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('value', d['value'], 'ms', d['ms_per_step'], 'frac', d['roofline']['frac'], 'search', d['search']['playouts_per_s'] if d['search'] else None, 'leaf', d['leaf_search']['playouts_per_s'] if d['leaf_search'] else None, 'clk', d['clocks'])"
timeout 400 ncu --set full --clock-control none --import-source on -k regex:playouts_kernel -s 3 -c 1 -o gpurun_out/prof_$TAG python bench.py --steps 2 --warmup 3 --no-search --no-cpu > /dev/null 2>&1; echo "ncu rc=$?"
