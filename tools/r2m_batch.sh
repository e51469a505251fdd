export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
bash tools/leaf_debug.sh r2m
timeout 600 python -m pytest tests -m gpu -q --timeout 200 --timeout_method=thread -k "leaf or search or pinned" > gpurun_out/r2m_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/r2m_pytest.log
timeout 200 python tools/leaf_probe.py > gpurun_out/r2m_leaf_probe.txt 2>&1; cat gpurun_out/r2m_leaf_probe.txt
timeout 400 python bench.py > gpurun_out/r2m_bench.json 2> gpurun_out/r2m_bench.err; echo "bench rc=$?"
python -c "import json;d=json.loads(open('gpurun_out/r2m_bench.json').read().splitlines()[-1]); print('value', d['value'], 'e2e', d['e2e']['value'], 'leaf', d['leaf_search']['iterations'], d['leaf_search']['playouts_per_s'], 'block', d['search']['playouts_per_s'], 'tree', d['tree_search']['playouts_per_s'])"
