#!/usr/bin/env python
"""Per-cell (V, S) geomean of cuBLAS Hgemm time / our single-call time from bench detail files."""
import collections
import json
import math
import sys

g = lambda v: math.exp(sum(math.log(t) for t in v) / len(v))
for f in sys.argv[1:]:
    a = json.load(open(f))["problems"]
    for op in ("sddmm", "spmm"):
        cell = collections.defaultdict(list)
        for x in a:
            cell[(x["V"], x["S"])].append(x["hgemm_us"] / x[op + "_us_warm"])
        print(f.split("/")[-1][:18], op, " ".join("%d/%.2f:%.2f" % (k[0], k[1], g(v)) for k, v in sorted(cell.items())))
