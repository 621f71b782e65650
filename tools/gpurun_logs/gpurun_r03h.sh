#!/bin/bash
# r03h: launch lists (single problems + the batched bench step) of the search-based dense SDDMM
for P in "512 512 64 2 0.9" "512 512 64 2 0.5" "2048 1024 256 2 0.5" "512 2048 64 8 0.5"; do
  set -- $P
  T=${1}_${2}_${3}_${4}_${5}
  timeout 300 ncu --metrics gpu__time_duration.sum,sm__cycles_active.avg,smsp__inst_executed.sum --clock-control none --csv --log-file gpurun_out/r03h_launch_$T.csv \
    python tools/one_problem.py --op sddmm --M $1 --K $2 --N $3 --V $4 --S $5 --reps 3 > /dev/null 2>&1
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"batched|dense" -c 60 --csv --log-file gpurun_out/r03h_step.csv \
  python bench.py --steps 1 --warmup 1 --no-baselines --no-cpu --no-e2e > /dev/null 2>&1
