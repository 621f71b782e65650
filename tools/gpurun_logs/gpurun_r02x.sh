#!/bin/bash
# r02x: harness validation of the multi-rank path on a 1-GPU box: `bench.py --gpus 2` spawns 2 ranks
# (torchrun), both on cuda:0 over gloo (VS_BENCH_HARNESS_TEST=1): plan, shards, gathers, max-over-ranks,
# JSON line.  Timings are NOT measurements (two ranks share one GPU).
VS_BENCH_HARNESS_TEST=1 timeout 1200 python bench.py --gpus 2 --steps 1 --warmup 1 --no-cpu > gpurun_out/r02x_c5_ws2.json 2> gpurun_out/r02x_c5_ws2.err
echo "rc=$?" >> gpurun_out/r02x_c5_ws2.err
VS_BENCH_HARNESS_TEST=1 timeout 900 python bench.py --gpus 2 --impl reference --steps 1 --warmup 0 > gpurun_out/r02x_ref_ws2.json 2> gpurun_out/r02x_ref_ws2.err
VS_BENCH_HARNESS_TEST=1 timeout 900 python bench.py --gpus 2 --workload dlmc_layer --steps 3 --warmup 3 --no-cpu --no-baselines > gpurun_out/r02x_dlmc_ws2.json 2> gpurun_out/r02x_dlmc_ws2.err
tail -3 gpurun_out/r02x_c5_ws2.err; head -c 1500 gpurun_out/r02x_c5_ws2.json
