export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
tools/gpu_batch.sh r2j "pinned or pool_full or hosted or ln_table" "" 0
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o /tmp/leaf_hang tools/leaf_hang.cu
for cfg in "8 400 3" "128 200 3"; do timeout 30 /tmp/leaf_hang $cfg >> gpurun_out/r2j_leaf_hang.txt 2>&1; echo "rc=$? $cfg" >> gpurun_out/r2j_leaf_hang.txt; done
cat gpurun_out/r2j_leaf_hang.txt
tools/sanitize.sh r2j
