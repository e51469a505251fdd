export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -q --timeout 200 --timeout_method=thread -k "leaf" > gpurun_out/r2p_pytest.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/r2p_pytest.log
tools/selfplay_round.sh r2p 32 500 tree
BENCH_DEBUG=1 timeout 4000 python bench.py --selfplay 32 --h2h --h2h-schemes hosted-hybrid,hosted --move-ms 500 --c-uct 0.25 > gpurun_out/r2p_h2h32_hostedhybrid_vs_hosted.json 2> gpurun_out/r2p_h2h.err
echo "h2h rc=$?"; python -c "import json;d=json.loads(open('gpurun_out/r2p_h2h32_hostedhybrid_vs_hosted.json').read().splitlines()[-1]); print(d['results'], d['win_pct'], d['mean_disc_diff'])"
