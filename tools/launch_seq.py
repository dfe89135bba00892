#!/usr/bin/env python
"""Print the kernel sequence (name, us, grid) of one Kalman update of a step from an ncu launch list:
  python tools/launch_seq.py launches.csv [step_index] [update_index]"""
import csv
import re
import sys


def load(path):
    rows = list(csv.reader(open(path)))
    hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hi]
    ki, vi, gi = h.index("Kernel Name"), h.index("Metric Value"), h.index("Grid Size")
    seq = []
    for r in rows[hi + 1:]:
        name = r[ki]
        m = re.search(r"dgemm_kernel<(\w+), (\w+), (\w+), (\w+), (\w+), (\w+), fekf::(\w+)", name)
        short = ("dgemm<%s,%s,%s>" % (m.group(1), m.group(2), m.group(7))) if m else \
            re.sub(r"\(.*", "", name).replace("void ", "").replace("fekf::", "").replace("<fekf::EmbW<25, 50, 100, 0>>", "")
        seq.append((short, float(r[vi].replace(",", "")) / 1e3, r[gi]))
    return seq


if __name__ == "__main__":
    seq = load(sys.argv[1])
    step = int(sys.argv[2]) if len(sys.argv) > 2 else 1
    upd = int(sys.argv[3]) if len(sys.argv) > 3 else 1
    ends = [i for i, (n, _, _) in enumerate(seq) if n == "metrics_kernel"]
    a = ends[step - 1] + 1 if step > 0 else 0
    b = ends[step] + 1
    ups, cur = [], []
    for x in seq[a:b]:
        cur.append(x)
        if x[0] == "kf_vec_kernel":
            ups.append(cur)
            cur = []
    for n, v, g in ups[upd]:
        print("%-34s %9.1f %s" % (n, v, g))
    print("update total %.1f us" % sum(v for _, v, _ in ups[upd]))
