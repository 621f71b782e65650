#!/bin/bash
# r04x: chain-schedule stream priority and schedule re-sweep with the dense-tile SDDMM (2 runs each)
A="--no-cpu --no-e2e --no-baselines --steps 20"
for r in 1 2; do
for pr in sddmm none first encode; do
  timeout 300 python bench.py $A --priority $pr > gpurun_out/r04x_$pr.json 2> gpurun_out/r04x_$pr.err
  echo "$pr $(grep classes_ms gpurun_out/r04x_$pr.err)" >> gpurun_out/r04x_summary.txt
done
done
cat gpurun_out/r04x_summary.txt
