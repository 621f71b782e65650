#!/bin/bash
# r04i: dense-tile SDDMM rule K >= 128 vs K >= 256 (1-stage ring, 4 CTAs/SM), batched classes + per-cell, 2 runs
A="--no-cpu --no-e2e --steps 20"
for r in 1 2; do
for v in default k128; do
  if [ $v = default ]; then L=paper_conf_sc_chenqldx21_b200/libvs.so; else L=build/variants/libvs_$v.so; fi
  VS_LIB_PATH=$L timeout 600 python bench.py $A > gpurun_out/r04i_$v.json 2> gpurun_out/r04i_$v.err
  cp gpurun_out/bench_detail.json gpurun_out/r04i_${v}_${r}_detail.json
  echo "$v $(grep classes_ms gpurun_out/r04i_$v.err)" >> gpurun_out/r04i_summary.txt
done
done
cat gpurun_out/r04i_summary.txt
