#!/bin/bash
# r04n: dense-tile SDDMM phase timing (clock64 per CTA, -DVS_SD_TIMING=1 build)
export VS_LIB_PATH=build/variants/libvs_sdt.so
for P in "2048 1024 256 2 0.5" "512 512 256 2 0.5" "2048 1024 256 8 0.5" "2048 1024 256 2 0.9"; do
  echo "== single $P" >> gpurun_out/r04n_timing.txt
  timeout 300 python tools/sd_timing.py $P >> gpurun_out/r04n_timing.txt 2>&1
done
echo "== batch (DLMC K=256, V=2, S .5/.7)" >> gpurun_out/r04n_timing.txt
timeout 300 python tools/sd_timing.py batch >> gpurun_out/r04n_timing.txt 2>&1
cat gpurun_out/r04n_timing.txt
unset VS_LIB_PATH
timeout 600 python -m pytest tests/test_gpu_dense.py tests/test_gpu_parity.py tests/test_gpu_coverage.py tests/test_gpu_batched.py -q -x -k "sddmm or batched" > gpurun_out/r04n_tests.log 2>&1; echo "rc=$?" >> gpurun_out/r04n_tests.log
A="--no-cpu --no-e2e --steps 20"
for r in 1 2; do
  timeout 600 python bench.py $A > gpurun_out/r04n_bench.json 2> gpurun_out/r04n_bench.err
  cp gpurun_out/bench_detail.json gpurun_out/r04n_${r}_detail.json
  echo "$(grep classes_ms gpurun_out/r04n_bench.err)" >> gpurun_out/r04n_summary.txt
done
cat gpurun_out/r04n_summary.txt; tail -n 2 gpurun_out/r04n_tests.log
