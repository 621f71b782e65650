set -x
mkdir -p build
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/gather_bench tools/gather_bench.cu && timeout 300 ./build/gather_bench > gpurun_out/e_gather.jsonl 2>&1; echo gather rc=$?
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv >> gpurun_out/e_gather_clocks.txt
