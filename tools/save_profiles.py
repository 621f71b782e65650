"""Copies one round's ncu evidence from gpurun_out/ into profiles/ (launch list summary, --set
full summaries, per-launch DRAM traffic scaled to the step) -- usage: save_profiles.py TAG BENCH_JSON"""
import json
import os
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
tag, bench = sys.argv[1], sys.argv[2]
g = os.path.join(ROOT, "gpurun_out")
pr = os.path.join(ROOT, "profiles")
d = json.loads(open(bench).read().strip().splitlines()[-1])
lm = subprocess.run([sys.executable, os.path.join(ROOT, "tools", "ncu_summary.py"), "launches",
                     os.path.join(g, f"launches_{tag}.csv")], capture_output=True, text=True).stdout
k = d["kernels"]
with open(os.path.join(pr, f"{tag}_launches.md"), "w") as f:
    f.write(f"# {tag} — ncu launch list of the batched bench step (dlmc_layer, 144 problems)\n\n")
    f.write("Command: tools/profile_round.sh (ncu --metrics gpu__time_duration.sum --clock-control none "
            "-k regex:batched -c 60: two full steps of 30 launches, the chains schedule then the phases schedule). Per-launch times are cold-cache and serialised: compare shares. "
            "Live in-graph CUDA-event times of the same step (bench.py): "
            + ", ".join(f"{c} {v['ms_per_step']:.3f} ms" for c, v in k.items())
            + f" per step; step {d['ms_per_step']:.3f} ms = {d['value']:.2f} TFLOP/s.\n\n")
    f.write(lm)
shutil.copy(os.path.join(g, f"launches_{tag}.csv"), os.path.join(pr, f"{tag}_launches.csv"))
t = {}
for kk in ["spmm_cp_batched", "sddmm_batched", "encode_count_batched", "encode_compact_batched"]:
    src = os.path.join(g, f"full_{tag}_{kk}.md")
    if os.path.exists(src):
        shutil.copy(src, os.path.join(pr, f"{tag}_full_{kk}.md"))
    tj = os.path.join(g, f"traffic_{tag}_{kk}.json")
    if os.path.exists(tj):
        t.update(json.load(open(tj)))
lp = d["roofline"]  # launches per class from the bench line
lpc = {c: v["launches_per_step"] for c, v in k.items()}
out = {"dlmc_layer:spmm": t.get("spmm_cp_batched_kernel", 0) * lpc["spmm"],
       "dlmc_layer:sddmm": t.get("sddmm_batched_kernel", 0) * lpc["sddmm"],
       "dlmc_layer:encode": (t.get("encode_count_batched_kernel", 0) + t.get("encode_compact_batched_kernel", 0))
       * (lpc["encode"] // 3),
       "per_launch_dram_bytes_ncu_set_full": t,
       "note": f"{tag}: DRAM read+write bytes per launch from ncu --set full (first 3 launches of each "
               "batched kernel class, cold caches) x launches per step of the class; "
               f"profiles/{tag}_full_*.md"}
json.dump(out, open(os.path.join(pr, "ncu_traffic.json"), "w"), indent=1)
shutil.copy(bench, os.path.join(pr, f"{tag}_bench.json"))
print(open(os.path.join(pr, f"{tag}_launches.md")).read())
