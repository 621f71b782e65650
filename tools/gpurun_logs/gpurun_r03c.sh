#!/bin/bash
# r03c: dense-tile SDDMM with the warp-chunk vote sampling: dense SDDMM suite + bench
timeout 600 python -m pytest tests/test_gpu_dense.py tests/test_gpu_parity.py -q -x -k sddmm > gpurun_out/r03c_dense.log 2>&1; echo "rc=$?" >> gpurun_out/r03c_dense.log
timeout 600 python bench.py --no-cpu --no-e2e --steps 20 > gpurun_out/r03c_bench.json 2> gpurun_out/r03c_bench.err
cp gpurun_out/bench_detail.json gpurun_out/r03c_detail.json
python -c "import json;d=json.loads(open('gpurun_out/r03c_bench.json').read().strip().splitlines()[-1]);print(round(d['ms_per_step'],4), {k:round(x['ms_per_step'],4) for k,x in d['kernels'].items()})" > gpurun_out/r03c_summary.txt 2>&1
tail -n 3 gpurun_out/r03c_dense.log gpurun_out/r03c_summary.txt; tail -n 5 gpurun_out/r03c_bench.err
