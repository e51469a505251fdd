export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
V="build/variants/libmcts_base.so build/variants/libmcts_ls2m4.so build/variants/libmcts_ls4m4.so build/variants/libmcts_ls8m4.so build/variants/libmcts_ls4.so build/variants/libmcts_ls16m4.so build/variants/libmcts_base.so"
tools/gpu_batch.sh r2i "pinned or pool or hosted" "$V" 0
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o /tmp/leaf_hang tools/leaf_hang.cu
for cfg in "128 200 2" "128 200 1" "128 200 0" "8 400 2" "512 100 2"; do timeout 30 /tmp/leaf_hang $cfg >> gpurun_out/r2i_leaf_hang.txt 2>&1; echo "rc=$? $cfg" >> gpurun_out/r2i_leaf_hang.txt; done
cat gpurun_out/r2i_leaf_hang.txt
tools/int_peaks_run.sh
tools/sanitize.sh r2i
