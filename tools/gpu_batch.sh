#!/bin/bash
# A batch of checks on the GPU box (run under gpurun): targeted tests, variant
# bench, bench line, sanitizers, integer peaks with clocks, NEXT-1 head-to-head.
# usage: tools/gpu_batch.sh TAG "pytest -k expr" "variant libs..." H2H_GAMES
TAG=$1; K=$2; VARS=$3; GAMES=${4:-0}
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
if [ -n "$K" ]; then
  timeout 900 python -m pytest tests -m gpu -q --timeout 300 --timeout_method=thread -k "$K" > gpurun_out/${TAG}_pytest.log 2>&1
  echo "pytest rc=$?"; tail -2 gpurun_out/${TAG}_pytest.log
fi
if [ -n "$VARS" ]; then
  nvcc -O2 -o /tmp/variant_bench tools/variant_bench.cu -ldl -Wno-deprecated-gpu-targets
  timeout 300 /tmp/variant_bench $VARS > gpurun_out/${TAG}_variants.txt 2>&1; cat gpurun_out/${TAG}_variants.txt
fi
timeout 400 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err; echo "bench rc=$?"
python -c "import json;d=json.loads(open('gpurun_out/${TAG}_bench.json').read().splitlines()[-1]); print('value', d['value'], 'e2e', d['e2e']['value'], 'frac', d['roofline']['frac'], d['roofline']['frac_executed'])"
if [ "$GAMES" -gt 0 ]; then
  BENCH_DEBUG=1 timeout $(( GAMES * 120 + 300 )) python bench.py --selfplay $GAMES --h2h --h2h-schemes hosted-hybrid,hosted \
    --move-ms 500 --c-uct 0.25 > gpurun_out/${TAG}_h2h_hostedhybrid_vs_hosted.json 2> gpurun_out/${TAG}_h2h.err
  echo "h2h rc=$?"; python -c "import json;d=json.loads(open('gpurun_out/${TAG}_h2h_hostedhybrid_vs_hosted.json').read().splitlines()[-1]); print(d['results'], d['win_pct'], d['mean_disc_diff'])"
fi
