#!/bin/bash
# r03l: launch list of the batched bench step (v5 dense SDDMM)
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"batched|dense" -c 400 --csv --log-file gpurun_out/r03l_step.csv \
  python bench.py --steps 1 --warmup 1 --no-baselines --no-cpu --no-e2e > /dev/null 2>&1
