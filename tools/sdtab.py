#!/usr/bin/env python
"""Prints per-problem SDDMM / SpMM single-call times from a bench detail file (tuning aid)."""
import json
import sys

d = json.load(open(sys.argv[1]))
ns = [int(x) for x in (sys.argv[2].split(",") if len(sys.argv) > 2 else ["64", "256"])]
tot = {}
for p in d["problems"]:
    tot.setdefault(p["V"], [0.0, 0.0])
    tot[p["V"]][0] += p["sddmm_us_warm"]
    tot[p["V"]][1] += p["spmm_us_warm"]
    if p["N"] in ns:
        print(p["M"], p["K"], p["N"], p["V"], p["S"], "sddmm %.1f spmm %.1f hgemm %.1f" % (
            p["sddmm_us_warm"], p["spmm_us_warm"], p["hgemm_us"]))
print("sum per V (sddmm, spmm us):", {k: (round(a, 1), round(b, 1)) for k, (a, b) in tot.items()})
