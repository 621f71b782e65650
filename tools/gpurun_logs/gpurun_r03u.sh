#!/bin/bash
# r03u: persistent dense SDDMM, 16-byte col_idx store pass
A="--no-cpu --no-e2e --no-baselines --steps 20"
timeout 600 python -m pytest tests/test_gpu_dense.py tests/test_gpu_parity.py tests/test_gpu_coverage.py -q -x -k sddmm > gpurun_out/r03u_tests.log 2>&1; echo "rc=$?" >> gpurun_out/r03u_tests.log
timeout 300 python bench.py $A > gpurun_out/r03u_bench.json 2> gpurun_out/r03u_bench.err
cp gpurun_out/bench_detail.json gpurun_out/r03u_detail.json
grep classes_ms gpurun_out/r03u_bench.err; tail -n 2 gpurun_out/r03u_tests.log
