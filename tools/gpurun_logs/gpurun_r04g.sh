#!/bin/bash
# r04g: dense-tile SDDMM, 1 stage + guided searches + fused row_ptr round trip + 8-window store rounds
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/r04g_gputest.log 2>&1; echo "rc=$?" >> gpurun_out/r04g_gputest.log
A="--no-cpu --no-e2e --steps 20"
for r in 1 2; do
  timeout 600 python bench.py $A > gpurun_out/r04g_bench.json 2> gpurun_out/r04g_bench.err
  cp gpurun_out/bench_detail.json gpurun_out/r04g_detail.json
  echo "$(grep classes_ms gpurun_out/r04g_bench.err)" >> gpurun_out/r04g_summary.txt
done
cat gpurun_out/r04g_summary.txt; tail -n 2 gpurun_out/r04g_gputest.log
