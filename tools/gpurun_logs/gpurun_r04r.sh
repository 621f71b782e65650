#!/bin/bash
# r04r: SDDMM gather launch with / without programmatic dependent launch after the dense-tile launch: DLMC batch + per-cell
A="--no-cpu --no-e2e --steps 20"
for v in default nopdl; do
  if [ $v = default ]; then L=paper_conf_sc_chenqldx21_b200/libvs.so; else L=build/variants/libvs_$v.so; fi
  VS_LIB_PATH=$L timeout 600 python bench.py $A > gpurun_out/r04r_$v.json 2> gpurun_out/r04r_$v.err
  cp gpurun_out/bench_detail.json gpurun_out/r04r_${v}_detail.json
  echo "$v $(grep classes_ms gpurun_out/r04r_$v.err)" >> gpurun_out/r04r_summary.txt
done
cat gpurun_out/r04r_summary.txt
