#!/bin/bash
# r03m: dense-tile SDDMM with 64-row units, 1 stage, 8 CTAs per SM, fused row_ptr round trip
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/r03m_gputest.log 2>&1; echo "rc=$?" >> gpurun_out/r03m_gputest.log
timeout 600 python bench.py --no-cpu --no-e2e --steps 20 > gpurun_out/r03m_bench.json 2> gpurun_out/r03m_bench.err
cp gpurun_out/bench_detail.json gpurun_out/r03m_detail.json
python -c "import json;d=json.loads(open('gpurun_out/r03m_bench.json').read().strip().splitlines()[-1]);print(round(d['ms_per_step'],4), {k:round(x['ms_per_step'],4) for k,x in d['kernels'].items()})" > gpurun_out/r03m_summary.txt 2>&1
tail -n 3 gpurun_out/r03m_gputest.log gpurun_out/r03m_summary.txt; tail -n 5 gpurun_out/r03m_bench.err
