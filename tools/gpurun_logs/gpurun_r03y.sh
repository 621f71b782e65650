#!/bin/bash
# r03y: per-problem single-call SDDMM: dense-tile build (default) vs gather-only build (VS_SDDMM_DENSE_CF=0)
A="--no-cpu --no-e2e --steps 20"
for v in default cf0; do
  if [ $v = default ]; then L=paper_conf_sc_chenqldx21_b200/libvs.so; else L=build/variants/libvs_$v.so; fi
  VS_LIB_PATH=$L timeout 600 python bench.py $A > gpurun_out/r03y_$v.json 2> gpurun_out/r03y_$v.err
  cp gpurun_out/bench_detail.json gpurun_out/r03y_${v}_detail.json
  echo "$v $(grep classes_ms gpurun_out/r03y_$v.err)" >> gpurun_out/r03y_summary.txt
done
cat gpurun_out/r03y_summary.txt
