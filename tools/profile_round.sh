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
# The batched step of bench.py: the eager sizing pass launches the single-problem kernels (and
# one dense SDDMM launch per eligible problem), then the step graph replays the batched ones.
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none \
  -k regex:"batched|dense" -c 400 --csv --log-file gpurun_out/launches_${TAG}_all.csv \
  python bench.py $ARGS > /dev/null 2>&1
# keep the batched step only: the launches after the eager pass's single-problem dense launches
python - "$TAG" <<'PY'
import csv, sys
tag = sys.argv[1]
rows = [r for r in csv.reader(open(f"gpurun_out/launches_{tag}_all.csv")) if r]
hdr_i = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
hdr, data = rows[hdr_i], rows[hdr_i + 1:]
k = hdr.index("Kernel Name")
first = next(i for i, r in enumerate(data) if "encode_count_batched" in r[k])
with open(f"gpurun_out/launches_{tag}.csv", "w", newline="") as f:
    w = csv.writer(f)
    w.writerow(hdr)
    ids = []
    for r in data[first:]:
        if r[0] not in ids:
            ids.append(r[0])
        w.writerow(r)
PY
for K in spmm_cp_batched sddmm_batched sddmm_dense encode_count_batched encode_compact_batched; do
  SKIP=0
  # the eager pass makes one single-problem dense SDDMM launch per eligible problem (48 at DLMC)
  if [ $K = sddmm_dense ]; then SKIP=48; fi
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:"$K" -s $SKIP -c 3 \
    -o /tmp/full_${TAG}_${K} python bench.py $ARGS > /tmp/ncu_${K}.log 2>&1
  python tools/ncu_summary.py full /tmp/full_${TAG}_${K}.ncu-rep > gpurun_out/full_${TAG}_${K}.md
  python tools/ncu_summary.py traffic /tmp/full_${TAG}_${K}.ncu-rep > gpurun_out/traffic_${TAG}_${K}.json
done
cp /tmp/full_${TAG}_sddmm_dense.ncu-rep gpurun_out/ 2>/dev/null
ls -la /tmp/*.ncu-rep
du -sh gpurun_out
