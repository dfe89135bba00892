#!/usr/bin/env python
"""One-screen summary of a bench.py JSON line."""
import json
import sys

d = json.loads([l for l in open(sys.argv[1]) if l.startswith("{")][-1])
print("images/s %.1f  ms/step %.2f  e2e %s" % (d["value"], d["ms_per_step"], d["e2e"] and round(d["e2e"]["value"], 1)))
r = d["roofline"]
print("P pass frac %.3f (alone %.3f)  split %s" % (r["frac"], r["standalone"]["frac"] if r.get("standalone") else -1,
                                                  {k: round(v, 2) for k, v in r["split_ms_per_pass"].items()}))
n = d.get("roofline_nets") or {}
print("nets %.2f TF/s frac %.3f alone %.2f ms/step" % (n.get("achieved", 0), n.get("frac", 0), n.get("ms_per_step_alone", 0)))
print("clocks", d["clocks"])
