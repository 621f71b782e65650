#!/bin/bash
# r03d: ncu of the dense-tile SDDMM on single problems (launch list + full set)
for P in "512 512 64 2 0.5" "2048 1024 256 2 0.5"; do
  set -- $P
  T=${1}_${2}_${3}_${4}_${5}
  timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r03d_launch_$T.csv \
    python tools/one_problem.py --op sddmm --M $1 --K $2 --N $3 --V $4 --S $5 --reps 3 > /dev/null 2>&1
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:sddmm_dense -c 1 -o gpurun_out/r03d_full_$T \
    python tools/one_problem.py --op sddmm --M $1 --K $2 --N $3 --V $4 --S $5 --reps 2 > gpurun_out/r03d_ncu_$T.log 2>&1
done
ls -la gpurun_out/ | grep r03d
