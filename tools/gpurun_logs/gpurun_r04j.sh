#!/bin/bash
# r04j: encode count pass, column steps in flight per warp: 2 (default) vs 4 vs 8
A="--no-cpu --no-e2e --no-baselines --steps 20"
for r in 1 2; do
for v in default cu4 cu8; do
  if [ $v = default ]; then L=paper_conf_sc_chenqldx21_b200/libvs.so; else L=build/variants/libvs_$v.so; fi
  VS_LIB_PATH=$L timeout 600 python bench.py $A > gpurun_out/r04j_$v.json 2> gpurun_out/r04j_$v.err
  echo "$v $(grep classes_ms gpurun_out/r04j_$v.err)" >> gpurun_out/r04j_summary.txt
done
done
cat gpurun_out/r04j_summary.txt
