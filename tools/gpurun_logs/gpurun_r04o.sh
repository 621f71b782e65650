#!/bin/bash
# r04o: C5 (1 GPU point) with the shipped library (dense-tile SDDMM launch in the path), and the
# multi-rank harness (2 ranks sharing cuda:0 over gloo, VS_BENCH_HARNESS_TEST=1: not measurements)
timeout 1500 python bench.py --workload c5 --steps 3 --warmup 3 > gpurun_out/r04o_c5.json 2> gpurun_out/r04o_c5.err; echo "rc=$?" >> gpurun_out/r04o_c5.err
VS_BENCH_HARNESS_TEST=1 timeout 1200 python bench.py --gpus 2 --steps 1 --warmup 1 --no-cpu > gpurun_out/r04o_c5_ws2.json 2> gpurun_out/r04o_c5_ws2.err; echo "rc=$?" >> gpurun_out/r04o_c5_ws2.err
VS_BENCH_HARNESS_TEST=1 timeout 900 python bench.py --gpus 2 --workload dlmc_layer --steps 3 --warmup 3 --no-cpu --no-baselines > gpurun_out/r04o_dlmc_ws2.json 2> gpurun_out/r04o_dlmc_ws2.err; echo "rc=$?" >> gpurun_out/r04o_dlmc_ws2.err
tail -n 2 gpurun_out/r04o_c5.err gpurun_out/r04o_c5_ws2.err gpurun_out/r04o_dlmc_ws2.err
