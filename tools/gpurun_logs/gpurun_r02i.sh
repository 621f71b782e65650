#!/bin/bash
# r02i: dense SDDMM v2b (8 stages, 1024-column units) -- tests, then per-problem calibration:
# the same bench with the gather-only and the dense-always builds (VS_DENSE_CF=0 / 1e9)
timeout 600 python -m pytest tests/test_gpu_dense.py tests/test_gpu_parity.py -x -q > gpurun_out/r02i_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r02i_tests.log
timeout 600 python bench.py --no-cpu --no-e2e --detail gpurun_out/cal_default.json > gpurun_out/r02i_bench.json 2> gpurun_out/r02i_bench.err
VS_LIB_PATH=build/variants/libvs_cf0.so timeout 600 python bench.py --no-cpu --no-e2e --detail gpurun_out/cal_cf0.json > gpurun_out/r02i_bench_cf0.json 2>&1
VS_LIB_PATH=build/variants/libvs_cfinf.so timeout 600 python bench.py --no-cpu --no-e2e --detail gpurun_out/cal_cfinf.json > gpurun_out/r02i_bench_cfinf.json 2>&1
tail -3 gpurun_out/r02i_tests.log
