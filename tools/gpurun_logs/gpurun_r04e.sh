#!/bin/bash
# r04e: final-state validation of round 2's shipped library (dense-tile SDDMM for K >= 256 + PDL):
# smoke, full GPU suite, compute-sanitizer memcheck + racecheck of the dense-tile SDDMM suites,
# default bench, sparsity-grid bench (per-V crossovers), ResNet-50 layer bench (C4)
CS=/usr/local/cuda/bin/compute-sanitizer
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r04e_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/r04e_smoke.log
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/r04e_gputest.log 2>&1; echo "rc=$?" >> gpurun_out/r04e_gputest.log
timeout 1200 $CS --tool memcheck --error-exitcode 9 python -m pytest tests/test_gpu_dense.py -q -x -k "sddmm and (unsorted or padded or mixed)" > gpurun_out/r04e_memcheck.log 2>&1; echo "rc=$?" >> gpurun_out/r04e_memcheck.log
timeout 1200 $CS --tool racecheck --error-exitcode 9 python -m pytest tests/test_gpu_dense.py -q -x -k "sddmm_dense_blocks and 256-256-256" > gpurun_out/r04e_racecheck.log 2>&1; echo "rc=$?" >> gpurun_out/r04e_racecheck.log
timeout 900 python bench.py > gpurun_out/r04e_bench.json 2> gpurun_out/r04e_bench.err
cp gpurun_out/bench_detail.json gpurun_out/r04e_detail.json
timeout 900 python bench.py --workload dlmc_grid --no-cpu --no-e2e > gpurun_out/r04e_grid.json 2> gpurun_out/r04e_grid.err
cp gpurun_out/bench_detail.json gpurun_out/r04e_grid_detail.json
timeout 900 python bench.py --workload rn50_layer --no-cpu --no-e2e > gpurun_out/r04e_rn50.json 2> gpurun_out/r04e_rn50.err
tail -n 2 gpurun_out/r04e_smoke.log gpurun_out/r04e_gputest.log gpurun_out/r04e_memcheck.log gpurun_out/r04e_racecheck.log
grep classes gpurun_out/r04e_bench.err gpurun_out/r04e_grid.err gpurun_out/r04e_rn50.err
