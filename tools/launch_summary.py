#!/usr/bin/env python
"""Summarise an ncu `--metrics gpu__time_duration.sum --csv` launch list per kernel (name, launches, ms, share)."""
import collections
import csv
import re
import sys


def summarise(path, per=1):
    rows = list(csv.reader(open(path)))
    hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hi]
    ki, vi = h.index("Kernel Name"), h.index("Metric Value")
    tot, cnt = collections.defaultdict(float), collections.Counter()
    for r in rows[hi + 1:]:
        name = r[ki]
        v = float(r[vi].replace(",", ""))
        m = re.search(r"dgemm_kernel<(\w+), (\w+), fekf::(\w+)", name)
        short = ("dgemm<%s,%s,%s>" % m.groups()) if m else re.sub(r"\(.*", "", name).replace("void ", "")
        tot[short] += v
        cnt[short] += 1
    T = sum(tot.values())
    out = ["| kernel | launches | total ms | share |", "|---|---|---|---|"]
    for k, v in sorted(tot.items(), key=lambda x: -x[1]):
        out.append(f"| `{k}` | {cnt[k]} | {v / 1e6 / per:.2f} | {100 * v / T:.1f}% |")
    out.append(f"\nTotal {T / 1e6 / per:.1f} ms")
    return "\n".join(out)


if __name__ == "__main__":
    print(summarise(sys.argv[1], float(sys.argv[2]) if len(sys.argv) > 2 else 1))
