#!/bin/bash
# r03f: ncu of the dense-tile SDDMM (warp-chunk sampling) on single problems
for P in "512 512 64 2 0.5" "512 512 64 2 0.9" "2048 1024 256 2 0.5"; do
  set -- $P
  T=${1}_${2}_${3}_${4}_${5}
  timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r03f_launch_$T.csv \
    python tools/one_problem.py --op sddmm --M $1 --K $2 --N $3 --V $4 --S $5 --reps 3 > /dev/null 2>&1
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:sddmm_dense -s 1 -c 1 -o gpurun_out/r03f_full_$T \
    python tools/one_problem.py --op sddmm --M $1 --K $2 --N $3 --V $4 --S $5 --reps 3 > gpurun_out/r03f_ncu_$T.log 2>&1
done
