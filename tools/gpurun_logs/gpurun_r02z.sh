#!/bin/bash
# r02z: ncu source-level (SASS) stall profile of the batched SDDMM and SpMM kernels of the bench step
ARGS="--steps 1 --warmup 1 --no-baselines --no-cpu --no-e2e --detail gpurun_out/prof_detail.json"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"sddmm_batched" -c 1 -o /tmp/src_sddmm python bench.py $ARGS > /tmp/ncu1.log 2>&1
ncu -i /tmp/src_sddmm.ncu-rep --page source --csv --print-source sass > gpurun_out/r02z_sddmm_sass.csv 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"spmm_cp_batched" -c 1 -o /tmp/src_spmm python bench.py $ARGS > /tmp/ncu2.log 2>&1
ncu -i /tmp/src_spmm.ncu-rep --page source --csv --print-source sass > gpurun_out/r02z_spmm_sass.csv 2>&1
ncu -i /tmp/src_sddmm.ncu-rep --page details --csv > gpurun_out/r02z_sddmm_details.csv 2>&1
ls -la gpurun_out/r02z*; head -3 gpurun_out/r02z_sddmm_sass.csv | cut -c1-400
