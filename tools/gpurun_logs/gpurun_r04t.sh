#!/bin/bash
# r04t: per-launch ring depth (1 stage for K <= 256, 3 stages above): dense suite, DLMC + rn50 benches
timeout 600 python -m pytest tests/test_gpu_dense.py tests/test_gpu_batched.py -q -x > gpurun_out/r04t_tests.log 2>&1; echo "rc=$?" >> gpurun_out/r04t_tests.log
timeout 600 python bench.py --no-cpu --no-e2e > gpurun_out/r04t_bench.json 2> gpurun_out/r04t_bench.err
cp gpurun_out/bench_detail.json gpurun_out/r04t_detail.json
timeout 900 python bench.py --workload rn50_layer --no-cpu --no-e2e > gpurun_out/r04t_rn50.json 2> gpurun_out/r04t_rn50.err
tail -n 2 gpurun_out/r04t_tests.log; grep classes gpurun_out/r04t_bench.err gpurun_out/r04t_rn50.err
