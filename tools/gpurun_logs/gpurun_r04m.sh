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
