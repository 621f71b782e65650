#!/bin/bash
# r02p: evidence run -- default bench (full), ncu launch list + --set full of the batched kernels,
# the paper's full sparsity grid with per-cell cuBLAS / cuSPARSE comparisons, C4 (rn50) and C5
timeout 900 python bench.py > gpurun_out/r02p_bench.json 2> gpurun_out/r02p_bench.err
timeout 1800 bash tools/profile_round.sh r02p > gpurun_out/r02p_profile.log 2>&1
timeout 1200 python bench.py --workload dlmc_grid --no-cpu --no-e2e --detail gpurun_out/r02p_grid_detail.json > gpurun_out/r02p_grid.json 2> gpurun_out/r02p_grid.err
timeout 900 python bench.py --workload rn50_layer --detail gpurun_out/r02p_rn50_detail.json > gpurun_out/r02p_rn50.json 2> gpurun_out/r02p_rn50.err
timeout 900 python bench.py --workload c5 --steps 3 --warmup 1 > gpurun_out/r02p_c5.json 2> gpurun_out/r02p_c5.err
ls -la gpurun_out | tail -30
