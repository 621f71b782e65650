#!/bin/bash
# r03k: fine warp-state sampling of the dense SDDMM (single problem, 512x512 V2 S.9 and 2048x1024x256 V2 S.5)
for P in "512 512 64 2 0.9" "2048 1024 64 2 0.5"; do
  set -- $P
  T=${1}_${2}_${3}_${4}_${5}
  timeout 300 ncu --set full --warp-sampling-interval 0 --clock-control none --import-source on -k regex:sddmm_dense -s 1 -c 1 -o gpurun_out/r03k_full_$T \
    python tools/one_problem.py --op sddmm --M $1 --K $2 --N $3 --V $4 --S $5 --reps 3 > gpurun_out/r03k_ncu_$T.log 2>&1
done
