#!/bin/bash
# r03r: batched-step launch list + one full ncu capture of the largest batched dense SDDMM launch
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"batched|dense" -c 400 --csv --log-file gpurun_out/r03r_step.csv \
  python bench.py --steps 1 --warmup 1 --no-baselines --no-cpu --no-e2e > /dev/null 2>&1
# eager pass = 144 single dense launches; batched step dense launches follow (4th batched one = large)
timeout 900 ncu --set full --warp-sampling-interval 2 --clock-control none --import-source on -k regex:sddmm_dense -s 147 -c 1 -o gpurun_out/r03r_full_batched \
  python bench.py --steps 1 --warmup 1 --no-baselines --no-cpu --no-e2e > gpurun_out/r03r_ncu.log 2>&1
