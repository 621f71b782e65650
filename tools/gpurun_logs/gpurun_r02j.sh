#!/bin/bash
# r02j: dense SDDMM v2b + dense SpMM -- dense tests, full GPU suite, default bench
timeout 600 python -m pytest tests/test_gpu_dense.py -x -q > gpurun_out/r02j_dense.log 2>&1
echo "rc=$?" >> gpurun_out/r02j_dense.log
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/r02j_gputest.log 2>&1
echo "rc=$?" >> gpurun_out/r02j_gputest.log
timeout 600 python bench.py --no-cpu --no-e2e > gpurun_out/r02j_bench.json 2> gpurun_out/r02j_bench.err
tail -3 gpurun_out/r02j_dense.log gpurun_out/r02j_gputest.log
