#!/bin/bash
# r02g: dense-tile SDDMM path -- dense tests, SDDMM suites, then the default bench
timeout 900 python -m pytest tests/test_gpu_dense.py -x -q > gpurun_out/r02g_dense.log 2>&1
echo "rc=$?" >> gpurun_out/r02g_dense.log
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/r02g_gputest.log 2>&1
echo "rc=$?" >> gpurun_out/r02g_gputest.log
timeout 600 python bench.py --no-cpu > gpurun_out/r02g_bench.json 2> gpurun_out/r02g_bench.err
tail -3 gpurun_out/r02g_dense.log gpurun_out/r02g_gputest.log
