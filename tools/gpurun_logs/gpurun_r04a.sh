#!/bin/bash
# r04a: dense SDDMM + PDL-overlapped gather launch: tests on default (CF64, any K), rule variants vs gather-only
timeout 600 python -m pytest tests -m gpu -q -x > gpurun_out/r04a_gputest.log 2>&1; echo "rc=$?" >> gpurun_out/r04a_gputest.log
A="--no-cpu --no-e2e --steps 20"
for v in default b d cf0; do
  if [ $v = default ]; then L=paper_conf_sc_chenqldx21_b200/libvs.so; else L=build/variants/libvs_$v.so; fi
  VS_LIB_PATH=$L timeout 600 python bench.py $A > gpurun_out/r04a_$v.json 2> gpurun_out/r04a_$v.err
  cp gpurun_out/bench_detail.json gpurun_out/r04a_${v}_detail.json
  echo "$v $(grep classes_ms gpurun_out/r04a_$v.err)" >> gpurun_out/r04a_summary.txt
done
cat gpurun_out/r04a_summary.txt; tail -n 2 gpurun_out/r04a_gputest.log
