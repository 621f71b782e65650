#!/bin/bash
# r05e: Fig. 20 analogue grid (sparse attention chain SDDMM -> softmax -> SpMM vs dense attention, 32 heads):
# l in {2048, 4096}, k in {64, 256}, S in {0.9, 0.95, 0.98}
for l in 2048 4096; do for k in 64 256; do for s in 0.9 0.95 0.98; do
  W=attention_l${l}_k${k}_s${s}
  timeout 300 python bench.py --workload $W --steps 10 --warmup 3 > gpurun_out/r05e_$W.json 2> gpurun_out/r05e_$W.err
done; done; done
python - <<'PY'
import glob, json
rows = []
for f in sorted(glob.glob("gpurun_out/r05e_attention_*.json")):
    t = open(f).read().strip().splitlines()
    if not t:
        continue
    d = json.loads(t[-1])
    rows.append((d["config"].get("workload"), round(d["ms_per_step"], 4), d.get("dense_attention_ms"), d.get("speedup_vs_dense"), d.get("stages_ms") or d.get("kernels")))
for r in rows:
    print(r)
PY
