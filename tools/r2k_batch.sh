export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o /tmp/leaf_hang tools/leaf_hang.cu
for cfg in "8 400 3" "128 200 0" "128 1000 0" "512 300 0"; do timeout 30 /tmp/leaf_hang $cfg >> gpurun_out/r2k_leaf_hang.txt 2>&1; echo "rc=$? $cfg" >> gpurun_out/r2k_leaf_hang.txt; done
cat gpurun_out/r2k_leaf_hang.txt
bash tools/leaf_debug.sh r2k
timeout 600 python -m pytest tests -m gpu -q --timeout 200 --timeout_method=thread -k "leaf or search" > gpurun_out/r2k_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/r2k_pytest.log
timeout 200 python tools/leaf_probe.py > gpurun_out/r2k_leaf_probe.txt 2>&1; cat gpurun_out/r2k_leaf_probe.txt
