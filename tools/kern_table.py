#!/usr/bin/env python
"""Table of an ncu --metrics --csv log: one line per launch (kernel, grid, metrics)."""
import csv
import sys

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 5]
h = rows[0]
ki, mi, vi, gi, ii = (h.index(k) for k in ("Kernel Name", "Metric Name", "Metric Value", "Grid Size", "ID"))
cur, order = {}, []
for r in rows[1:]:
    key = (r[ii], r[ki].replace("void ", "")[:44], r[gi])
    if key not in cur:
        cur[key] = {}
        order.append(key)
    cur[key][r[mi].split(".")[0]] = r[vi]
for k in order:
    print("%-44s %-14s %s" % (k[1], k[2], " ".join("%s=%s" % (a.replace("__", ":"), b) for a, b in cur[k].items())))
