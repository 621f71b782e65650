#!/bin/bash
# r03b: new 128x128-unit dense-tile SDDMM (VS_SDDMM_DENSE_CF=64 default): SDDMM suites, full GPU suite, bench
timeout 600 python -m pytest tests/test_gpu_dense.py -q -x -k sddmm > gpurun_out/r03b_dense.log 2>&1; echo "rc=$?" >> gpurun_out/r03b_dense.log
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/r03b_gputest.log 2>&1; echo "rc=$?" >> gpurun_out/r03b_gputest.log
timeout 600 python bench.py --no-cpu --no-e2e --steps 20 > gpurun_out/r03b_bench.json 2> gpurun_out/r03b_bench.err
python -c "import json;d=json.loads(open('gpurun_out/r03b_bench.json').read().strip().splitlines()[-1]);print(round(d['ms_per_step'],4), {k:round(x['ms_per_step'],4) for k,x in d['kernels'].items()})" > gpurun_out/r03b_summary.txt 2>&1
tail -n 3 gpurun_out/r03b_dense.log gpurun_out/r03b_gputest.log gpurun_out/r03b_summary.txt; tail -n 5 gpurun_out/r03b_bench.err
