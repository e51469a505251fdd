#!/bin/bash
# Equal-C self-play sets vs the all-core CPU oracle MCTS (run under gpurun).
# usage: tools/selfplay_round.sh TAG GAMES MS SCHEME [SCHEME ...]
TAG=$1; GAMES=$2; MS=$3; shift 3
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
for S in "$@"; do
  BENCH_DEBUG=1 timeout $(( GAMES * 120 + 300 )) python bench.py --selfplay $GAMES --move-ms $MS --sp-scheme $S \
    --c-uct 0.25 > gpurun_out/${TAG}_selfplay${GAMES}_${S}_equalC.json 2> gpurun_out/${TAG}_selfplay_${S}.err
  echo "selfplay $S rc=$?"
  python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().splitlines()[-1]); print(sys.argv[2], d['results'], round(d['win_pct'],1), 'refused', d.get('gpu_refused_expansions'), 'fill', round(d.get('gpu_pool_max_fill') or 0, 4))" gpurun_out/${TAG}_selfplay${GAMES}_${S}_equalC.json $S
done
