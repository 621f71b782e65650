#!/bin/bash
# r04f: dense-tile SDDMM with a 1-stage ring (4 CTAs per SM, TMEM-bound) vs 2 stages (3 CTAs per SM)
timeout 600 env VS_LIB_PATH=build/variants/libvs_st1.so python -m pytest tests/test_gpu_dense.py -q -x -k sddmm > gpurun_out/r04f_tests.log 2>&1; echo "rc=$?" >> gpurun_out/r04f_tests.log
A="--no-cpu --no-e2e --steps 20"
for r in 1 2; do
for v in default st1; do
  if [ $v = default ]; then L=paper_conf_sc_chenqldx21_b200/libvs.so; else L=build/variants/libvs_$v.so; fi
  VS_LIB_PATH=$L timeout 600 python bench.py $A > gpurun_out/r04f_$v.json 2> gpurun_out/r04f_$v.err
  cp gpurun_out/bench_detail.json gpurun_out/r04f_${v}_detail.json
  echo "$v $(grep classes_ms gpurun_out/r04f_$v.err)" >> gpurun_out/r04f_summary.txt
done
done
cat gpurun_out/r04f_summary.txt; tail -n 2 gpurun_out/r04f_tests.log
