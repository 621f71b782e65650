#!/bin/bash
# r04c: 128-row dense-tile SpMM (K <= 512, decoded A tile resident) variants: SpMM suites + bench
for v in sp32 sp64; do
  VS_LIB_PATH=build/variants/libvs_$v.so timeout 900 python -m pytest tests -m gpu -q -x -k "spmm or batched or scatter or shard or transpose or attention or dense" > gpurun_out/r04c_tests_$v.log 2>&1; echo "rc=$?" >> gpurun_out/r04c_tests_$v.log
done
A="--no-cpu --no-e2e --steps 20"
for v in default sp32 sp64; do
  if [ $v = default ]; then L=paper_conf_sc_chenqldx21_b200/libvs.so; else L=build/variants/libvs_$v.so; fi
  VS_LIB_PATH=$L timeout 600 python bench.py $A > gpurun_out/r04c_$v.json 2> gpurun_out/r04c_$v.err
  cp gpurun_out/bench_detail.json gpurun_out/r04c_${v}_detail.json
  echo "$v $(grep classes_ms gpurun_out/r04c_$v.err)" >> gpurun_out/r04c_summary.txt
done
cat gpurun_out/r04c_summary.txt; tail -n 2 gpurun_out/r04c_tests_*.log
