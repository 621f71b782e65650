#!/bin/bash
# r03q: dense-tile SDDMM with persistent warp-specialised dense SDDMM
timeout 600 python -m pytest tests -m gpu -q -x > gpurun_out/r03q_gputest.log 2>&1; echo "rc=$?" >> gpurun_out/r03q_gputest.log
timeout 600 python bench.py --no-cpu --no-e2e --steps 20 > gpurun_out/r03q_bench.json 2> gpurun_out/r03q_bench.err
cp gpurun_out/bench_detail.json gpurun_out/r03q_detail.json
python -c "import json;d=json.loads(open('gpurun_out/r03q_bench.json').read().strip().splitlines()[-1]);print(round(d['ms_per_step'],4), {k:round(x['ms_per_step'],4) for k,x in d['kernels'].items()})" > gpurun_out/r03q_summary.txt 2>&1
tail -n 3 gpurun_out/r03q_gputest.log gpurun_out/r03q_summary.txt; tail -n 5 gpurun_out/r03q_bench.err
