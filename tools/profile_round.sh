#!/bin/bash
# Runs on the GPU box (via gpurun) and leaves the ncu evidence for profiles/ in gpurun_out/:
#   launches_<tag>.csv    every kernel of one batched bench step with its device time
#                         (ncu --metrics gpu__time_duration.sum --clock-control none)
#   full_<tag>_<k>.md     ncu --set full summaries of the batched kernels (made on the box;
#                         the .ncu-rep files are kept only if small)
#   traffic_<tag>.json    dram bytes per launch of each batched kernel class
# Usage: bash tools/profile_round.sh <tag>
set -x
TAG=${1:-r01}
ARGS="--steps 1 --warmup 1 --no-baselines --no-cpu --no-e2e --detail gpurun_out/prof_detail.json"
# The batched step of bench.py: the warm-up replays the step graph once; kernels named
# *batched* belong to it (the eager sizing pass uses the single-problem
# kernels, which the regex excludes).
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none \
  -k regex:"batched" -c 60 --csv --log-file gpurun_out/launches_${TAG}.csv \
  python bench.py $ARGS > /dev/null 2>&1
for K in spmm_cp_batched sddmm_batched encode_count_batched encode_compact_batched; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:"$K" -c 3 \
    -o /tmp/full_${TAG}_${K} python bench.py $ARGS > /tmp/ncu_${K}.log 2>&1
  python tools/ncu_summary.py full /tmp/full_${TAG}_${K}.ncu-rep > gpurun_out/full_${TAG}_${K}.md
  python tools/ncu_summary.py traffic /tmp/full_${TAG}_${K}.ncu-rep > gpurun_out/traffic_${TAG}_${K}.json
done
ls -la /tmp/*.ncu-rep
du -sh gpurun_out
