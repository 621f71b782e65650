#!/bin/bash
# r02y: compute-sanitizer memcheck of the round-2 paths (scatter epilogue incl. symmetric memory,
# SPLIT=4 + permuted/duplicate col_idx coverage, batched), racecheck of the scatter tests; then the
# final default-config validation: smoke, full GPU suite, default bench
CS=/usr/local/cuda/bin/compute-sanitizer
timeout 1500 $CS --tool memcheck --error-exitcode 9 python -m pytest tests/test_gpu_scatter.py tests/test_gpu_batched.py -q -x > gpurun_out/r02y_memcheck_a.log 2>&1; echo "rc=$?" >> gpurun_out/r02y_memcheck_a.log
timeout 1500 $CS --tool memcheck --error-exitcode 9 python -m pytest tests/test_gpu_coverage.py -q -x -k "perm and (64-300 or 40-90)" > gpurun_out/r02y_memcheck_b.log 2>&1; echo "rc=$?" >> gpurun_out/r02y_memcheck_b.log
timeout 1500 $CS --tool racecheck --error-exitcode 9 python -m pytest tests/test_gpu_scatter.py -q -x -k "reassemble and 256" > gpurun_out/r02y_racecheck.log 2>&1; echo "rc=$?" >> gpurun_out/r02y_racecheck.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02y_smoke.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r02y_gputest.log 2>&1; echo "rc=$?" >> gpurun_out/r02y_gputest.log
timeout 900 python bench.py > gpurun_out/r02y_bench.json 2> gpurun_out/r02y_bench.err
tail -2 gpurun_out/r02y_memcheck_a.log gpurun_out/r02y_memcheck_b.log gpurun_out/r02y_racecheck.log gpurun_out/r02y_smoke.log gpurun_out/r02y_gputest.log
