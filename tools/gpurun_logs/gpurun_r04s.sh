#!/bin/bash
# r04s: final shipped state (dense-tile SDDMM for K >= 256, plain stream order): smoke, full GPU suite,
# default bench, C5 1-GPU point, sparsity grid, ResNet-50 layers, ncu profile round r05
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r04s_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/r04s_smoke.log
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/r04s_gputest.log 2>&1; echo "rc=$?" >> gpurun_out/r04s_gputest.log
timeout 900 python bench.py > gpurun_out/r04s_bench.json 2> gpurun_out/r04s_bench.err
cp gpurun_out/bench_detail.json gpurun_out/r04s_detail.json
timeout 1500 python bench.py --workload c5 --steps 3 --warmup 3 > gpurun_out/r04s_c5.json 2> gpurun_out/r04s_c5.err
timeout 900 python bench.py --workload dlmc_grid --no-cpu --no-e2e > gpurun_out/r04s_grid.json 2> gpurun_out/r04s_grid.err
cp gpurun_out/bench_detail.json gpurun_out/r04s_grid_detail.json
timeout 900 python bench.py --workload rn50_layer --no-cpu --no-e2e > gpurun_out/r04s_rn50.json 2> gpurun_out/r04s_rn50.err
bash tools/profile_round.sh r05 > gpurun_out/profile_r05.log 2>&1
tail -n 2 gpurun_out/r04s_smoke.log gpurun_out/r04s_gputest.log
grep classes gpurun_out/r04s_bench.err gpurun_out/r04s_grid.err gpurun_out/r04s_rn50.err
