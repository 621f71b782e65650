#!/bin/bash
# r03x: dense-tile SDDMM cost-model constant sweep (VS_SDDMM_DENSE_CF 32/64/128/256), DLMC batch, 2 runs each
A="--no-cpu --no-e2e --no-baselines --steps 20"
for r in 1 2; do
for v in cf32 default cf128 cf256; do
  if [ $v = default ]; then L=paper_conf_sc_chenqldx21_b200/libvs.so; else L=build/variants/libvs_$v.so; fi
  VS_LIB_PATH=$L timeout 300 python bench.py $A > gpurun_out/r03x_$v.json 2> gpurun_out/r03x_$v.err
  cp gpurun_out/bench_detail.json gpurun_out/r03x_${v}_detail.json
  echo "$v $(grep classes_ms gpurun_out/r03x_$v.err)" >> gpurun_out/r03x_summary.txt
done
done
cat gpurun_out/r03x_summary.txt
