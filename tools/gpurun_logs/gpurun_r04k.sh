#!/bin/bash
# r04k: single-call kernel durations (ncu launch list) of the shipped dense-tile SDDMM path
for P in "2048 1024 256 2 0.5" "2048 1024 256 8 0.5" "512 512 256 2 0.5" "2048 1024 256 2 0.98"; do
  set -- $P
  T=${1}_${2}_${3}_${4}_${5}
  timeout 300 ncu --metrics gpu__time_duration.sum,sm__cycles_active.avg --clock-control none --csv --log-file gpurun_out/r04k_launch_$T.csv \
    python tools/one_problem.py --op sddmm --M $1 --K $2 --N $3 --V $4 --S $5 --reps 3 > /dev/null 2>&1
done
