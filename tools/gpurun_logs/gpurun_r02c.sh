set -x
mkdir -p build
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build/gather_bench tools/gather_bench.cu && ./build/gather_bench > gpurun_out/gather_bench.jsonl 2>&1
for CP in 0 3; do
VS_SPMM_CP=$CP timeout 600 ncu --set full --clock-control none --import-source on -k regex:"spmm" -s 1 -c 1 -o /tmp/one_cp$CP python tools/one_problem.py --op spmm --M 2048 --K 1024 --N 256 --V 2 --S 0.5 > /tmp/ncu_$CP.log 2>&1
python tools/ncu_summary.py full /tmp/one_cp$CP.ncu-rep > gpurun_out/one_cp$CP.md
ncu -i /tmp/one_cp$CP.ncu-rep --page source --csv > gpurun_out/one_cp${CP}_source.csv 2>/dev/null
cp /tmp/one_cp$CP.ncu-rep gpurun_out/
done
cat gpurun_out/gather_bench.jsonl gpurun_out/one_cp0.md gpurun_out/one_cp3.md
