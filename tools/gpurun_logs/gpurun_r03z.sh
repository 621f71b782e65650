#!/bin/bash
# r03z: dense-tile SDDMM rule variants (shape rule K >= KMIN, density CF) vs gather-only: batched classes + per-cell single calls
A="--no-cpu --no-e2e --steps 20"
for v in cf0 a b c; do
  L=build/variants/libvs_$v.so
  VS_LIB_PATH=$L timeout 600 python bench.py $A > gpurun_out/r03z_$v.json 2> gpurun_out/r03z_$v.err
  cp gpurun_out/bench_detail.json gpurun_out/r03z_${v}_detail.json
  echo "$v $(grep classes_ms gpurun_out/r03z_$v.err)" >> gpurun_out/r03z_summary.txt
done
cat gpurun_out/r03z_summary.txt
