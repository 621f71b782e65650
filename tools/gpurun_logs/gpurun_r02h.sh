#!/bin/bash
# r02h: dense-tile SDDMM v2 (32-row units, flat sampled pass)
timeout 600 python -m pytest tests/test_gpu_dense.py -x -q > gpurun_out/r02h_dense.log 2>&1
echo "rc=$?" >> gpurun_out/r02h_dense.log
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/r02h_gputest.log 2>&1
echo "rc=$?" >> gpurun_out/r02h_gputest.log
timeout 600 python bench.py --no-cpu > gpurun_out/r02h_bench.json 2> gpurun_out/r02h_bench.err
tail -3 gpurun_out/r02h_dense.log gpurun_out/r02h_gputest.log
