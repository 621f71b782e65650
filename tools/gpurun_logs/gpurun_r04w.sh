#!/bin/bash
# r04w: 16-byte-load sortedness check in the gather kernels (dense-block windows): tests + DLMC bench x2
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/r04w_gputest.log 2>&1; echo "rc=$?" >> gpurun_out/r04w_gputest.log
for r in 1 2; do
  timeout 600 python bench.py --no-cpu --no-e2e --no-baselines --steps 20 > gpurun_out/r04w_bench.json 2> gpurun_out/r04w_bench.err
  echo "$(grep classes_ms gpurun_out/r04w_bench.err)" >> gpurun_out/r04w_summary.txt
done
cat gpurun_out/r04w_summary.txt; tail -n 2 gpurun_out/r04w_gputest.log
