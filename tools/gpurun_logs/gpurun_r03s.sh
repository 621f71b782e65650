#!/bin/bash
# r03s: persistent dense SDDMM role experiments: default vs no store pass (exp1) vs no search + no store (exp2)
A="--no-cpu --no-e2e --no-baselines --steps 20"
for v in default exp1 exp2; do
  if [ $v = default ]; then L=paper_conf_sc_chenqldx21_b200/libvs.so; else L=build/variants/libvs_$v.so; fi
  VS_LIB_PATH=$L timeout 300 python bench.py $A > gpurun_out/r03s_$v.json 2> gpurun_out/r03s_$v.err
  echo "$v $(grep classes_ms gpurun_out/r03s_$v.err)" >> gpurun_out/r03s_summary.txt
done
cat gpurun_out/r03s_summary.txt
