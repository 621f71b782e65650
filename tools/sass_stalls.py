#!/usr/bin/env python
"""Per-region stall-reason breakdown of an ncu source page (SASS) CSV (tuning aid).

  python tools/sass_stalls.py x.csv start end   # instruction index range (0-based rows)
"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
data = rows[2:]
a, b = int(sys.argv[2]), int(sys.argv[3])
cols = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
tot = {c: 0.0 for c in cols}
for r in data[a:b]:
    for c in cols:
        tot[c] += float(r[hdr.index(c)] or 0)
s = sum(tot.values())
print("region %d-%d samples %d" % (a, b, s))
for c, v in sorted(tot.items(), key=lambda x: -x[1])[:8]:
    print("  %-22s %5.1f%%" % (c, 100 * v / max(s, 1)))
