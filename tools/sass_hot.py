#!/usr/bin/env python
"""Hot SASS regions of one kernel from `ncu -i rep --page source --csv --print-source sass` output:
stall samples per window of instructions, and the hottest instructions with their top stall reasons."""
import csv
import sys
from collections import Counter


def main(path, kidx=0, win=100, top=30):
    rows = list(csv.reader(open(path)))
    ks = [i for i, r in enumerate(rows) if r and r[0] == "Kernel Name"] + [len(rows)]
    start, end = ks[kidx], ks[kidx + 1]
    hdr = rows[start + 1]
    data = [r for r in rows[start + 2:end] if r and r[0] != "Address"]
    si = hdr.index("Warp Stall Sampling (All Samples)")
    cols = [c for c in hdr if c.startswith("stall_") and "(Not" not in c]
    f = lambda r: float(r[si] or 0)
    tot = sum(f(r) for r in data)
    print(rows[start][1][:80], "samples", tot, "instructions", len(data))
    for b in range(0, len(data), win):
        s = sum(f(r) for r in data[b:b + win])
        if s / tot > 0.02:
            ops = Counter(r[1].split()[0] for r in data[b:b + win] if r[1] and not r[1].startswith("@"))
            print(f"  [{b:5d}] {100 * s / tot:5.1f}%  {ops.most_common(4)}")
    for i in sorted(sorted(range(len(data)), key=lambda i: -f(data[i]))[:top]):
        r = data[i]
        st = sorted(((float(r[hdr.index(c)] or 0), c[6:]) for c in cols), reverse=True)[:2]
        print(f"  {i:5d} {r[1][:70]:70s} {f(r):7.0f} {st}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 0)
