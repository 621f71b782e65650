#!/usr/bin/env python
"""Summarises an ncu source page (SASS) CSV: warp-stall samples per region (tuning aid).

  ncu -i rep.ncu-rep --page source --csv --print-source sass > x.csv; python tools/sass_regions.py x.csv [block]
"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
blk = int(sys.argv[2]) if len(sys.argv) > 2 else 40
hdr = rows[1]
i_src = hdr.index("Source")
i_st = hdr.index("Warp Stall Sampling (All Samples)")
i_ex = hdr.index("Instructions Executed")
data = rows[2:]
tot = sum(float(r[i_st] or 0) for r in data)
print("samples", tot, "instructions", sum(float(r[i_ex] or 0) for r in data))
acc = 0
start = 0
for i, r in enumerate(data):
    acc += float(r[i_st] or 0)
    if i % blk == blk - 1 or i == len(data) - 1:
        if acc > 0.01 * tot:
            srcs = [x[i_src].split()[0] if not x[i_src].startswith("@") else x[i_src].split()[1]
                    for x in data[start:i + 1]]
            keys = [s for s in srcs if s.split(".")[0] in ("UTMALDG", "UTCHMMA", "LDTM", "LDG", "STG", "LDS", "STS",
                                                         "SYNCS", "BAR", "EXIT", "VOTE", "SHFL", "ATOMS", "F2FP")]
            print("%4d-%4d %5.1f%%  %s" % (start, i, 100 * acc / tot, " ".join(sorted(set(keys)))))
        acc = 0
        start = i + 1
