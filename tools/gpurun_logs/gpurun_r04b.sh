#!/bin/bash
# r04b: shipped rule (dense SDDMM for K >= 256, density > V/32, PDL-overlapped gather): smoke, full GPU suite, default bench
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r04b_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/r04b_smoke.log
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/r04b_gputest.log 2>&1; echo "rc=$?" >> gpurun_out/r04b_gputest.log
timeout 900 python bench.py > gpurun_out/r04b_bench.json 2> gpurun_out/r04b_bench.err
cp gpurun_out/bench_detail.json gpurun_out/r04b_detail.json
tail -n 2 gpurun_out/r04b_smoke.log gpurun_out/r04b_gputest.log; grep classes gpurun_out/r04b_bench.err
