#!/bin/bash
# r02f: scatter / coverage tests, then C5 (1 GPU, strong-scaling point) and C4 (rn50) bench lines
timeout 900 python -m pytest tests/test_gpu_scatter.py tests/test_gpu_coverage.py tests/test_gpu_transpose.py tests/test_gpu_attention.py -x -q > gpurun_out/r02f_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r02f_tests.log
timeout 900 python bench.py --workload c5 --steps 3 --warmup 1 > gpurun_out/r02f_c5.json 2> gpurun_out/r02f_c5.err
timeout 900 python bench.py --workload rn50_layer > gpurun_out/r02f_rn50.json 2> gpurun_out/r02f_rn50.err
tail -2 gpurun_out/r02f_tests.log
