#!/bin/bash
# r04z: gather SDDMM resident CTAs per SM (VS_SDDMM_MINB 4 / 5 / 6) re-tuned with the dense-tile SDDMM taking K >= 256 blocks
A="--no-cpu --no-e2e --no-baselines --steps 20"
for r in 1 2; do
for v in default minb4 minb6; do
  if [ $v = default ]; then L=paper_conf_sc_chenqldx21_b200/libvs.so; else L=build/variants/libvs_$v.so; fi
  VS_LIB_PATH=$L timeout 300 python bench.py $A > gpurun_out/r04z_$v.json 2> gpurun_out/r04z_$v.err
  echo "$v $(grep classes_ms gpurun_out/r04z_$v.err)" >> gpurun_out/r04z_summary.txt
done
done
cat gpurun_out/r04z_summary.txt
