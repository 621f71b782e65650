#!/usr/bin/env python
"""Summarise ncu output into the tables committed under profiles/.

  python tools/ncu_summary.py launches gpurun_out/launches.csv   > profiles/rNN_launches.md
  python tools/ncu_summary.py full gpurun_out/prof.ncu-rep        > profiles/rNN_full.md
  python tools/ncu_summary.py traffic gpurun_out/prof.ncu-rep KEY  (prints JSON bytes/launch)
"""
from __future__ import annotations

import collections
import csv
import io
import json
import subprocess
import sys

NCU = "/usr/local/cuda/bin/ncu"

FULL_METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("lts__t_bytes.sum", "L2 bytes"),
    ("l1tex__t_bytes.sum", "L1 bytes"),
    ("lts__t_sector_hit_rate.pct", "L2 hit %"),
    ("l1tex__t_sector_hit_rate.pct", "L1 hit %"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps active %"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM thru %"),
    ("gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed", "mem thru %"),
    ("TPC.TriageCompute.sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed", "tensor pipe %"),
    ("sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active", "LSU issue %"),
    ("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "smem wavefronts"),
    ("l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "gld sectors"),
    ("l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum", "gld requests"),
    ("launch__registers_per_thread", "regs"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
]


def short(name: str) -> str:
    name = name.replace("void ", "")
    return name.split("(")[0]


def launches(path: str) -> str:
    rows = list(csv.reader(open(path)))
    hdr, data = None, []
    for r in rows:
        if r and r[0] == "ID":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            data.append(dict(zip(hdr, r)))
    agg = collections.OrderedDict()
    for d in data:
        k = short(d["Kernel Name"]).split("<")[0]
        agg.setdefault(k, []).append(float(d["Metric Value"]))
    tot = sum(sum(v) for v in agg.values())
    out = ["| kernel | launches | total µs | share | mean µs | max µs |", "|---|---|---|---|---|---|"]
    for k, v in agg.items():
        out.append(f"| {k} | {len(v)} | {sum(v)/1e3:.1f} | {sum(v)/tot:.3f} | {sum(v)/len(v)/1e3:.2f} | {max(v)/1e3:.2f} |")
    out.append(f"\n{len(data)} launches, {tot/1e3:.1f} µs total (ncu gpu__time_duration, serialised, cold caches).")
    return "\n".join(out)


def raw(path: str):
    txt = subprocess.run([NCU, "-i", path, "--page", "raw", "--csv"], capture_output=True,
                         text=True, check=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    hdr, units = rows[0], rows[1]
    return hdr, units, rows[2:]


def full(path: str) -> str:
    hdr, units, data = raw(path)
    col = {h: i for i, h in enumerate(hdr)}
    out = []
    stall_cols = [h for h in hdr if h.startswith("smsp__average_warps_issue_stalled_")
                  and h.endswith("_per_issue_active.ratio")]
    for d in data:
        out.append(f"### {short(d[col['Kernel Name']])}\n")
        out.append("| metric | value |\n|---|---|")
        for m, label in FULL_METRICS:
            if m in col:
                out.append(f"| {label} (`{m}`) | {d[col[m]]} {units[col[m]]} |")
        stalls = []
        for h in stall_cols:
            try:
                stalls.append((float(d[col[h]].replace(",", "")), h))
            except ValueError:
                pass
        stalls.sort(reverse=True)
        if stalls:
            out.append("\nTop stall reasons (warps stalled per issued instruction):\n")
            for v, h in stalls[:6]:
                name = h.replace("smsp__average_warps_issue_stalled_", "").replace("_per_issue_active.ratio", "")
                out.append(f"- {name}: {v:.2f}")
        out.append("")
    return "\n".join(out)


def traffic(path: str) -> dict:
    hdr, units, data = raw(path)
    col = {h: i for i, h in enumerate(hdr)}
    res = collections.defaultdict(list)
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
    for d in data:
        k = short(d[col["Kernel Name"]]).split("<")[0]
        b = 0.0
        for m in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
            b += float(d[col[m]].replace(",", "")) * scale.get(units[col[m]], 1)
        res[k].append(b)
    return {k: sum(v) / len(v) for k, v in res.items()}


if __name__ == "__main__":
    cmd, path = sys.argv[1], sys.argv[2]
    if cmd == "launches":
        print(launches(path))
    elif cmd == "full":
        print(full(path))
    elif cmd == "traffic":
        print(json.dumps(traffic(path), indent=1))
