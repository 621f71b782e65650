#!/bin/bash
# r02t: ncu A/B of the tcgen05 gather-ring SpMM (VS_SPMM_TC=1) against the shipped cp.async kernel
ARGS="--steps 1 --warmup 1 --no-baselines --no-cpu --no-e2e --detail gpurun_out/prof_detail.json"
VS_LIB_PATH=build/variants/libvs_stc.so timeout 900 ncu --set full --clock-control none -k regex:"spmm_tc_kernel" -c 3 \
  -o /tmp/full_r02t_spmm_tc python bench.py $ARGS > /tmp/ncu_tc.log 2>&1
python tools/ncu_summary.py full /tmp/full_r02t_spmm_tc.ncu-rep > gpurun_out/full_r02t_spmm_tc.md
VS_LIB_PATH=build/variants/libvs_stc.so timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"batched|spmm_tc" -c 60 --csv \
  --log-file gpurun_out/launches_r02t_tc.csv python bench.py $ARGS > /dev/null 2>&1
tail -3 /tmp/ncu_tc.log; ls -la gpurun_out | tail
