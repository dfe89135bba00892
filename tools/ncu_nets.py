#!/usr/bin/env python
"""Per-launch fp64 tensor-pipe utilisation and top stall reasons of ncu reports (`--set full`):
`ncu_nets.py rep1.ncu-rep [rep2 ...]`.  DMMA share = smsp dmma sub-pipe active cycles / SM cycles elapsed."""
import csv
import io
import subprocess
import sys


def main(paths):
    for path in paths:
        out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
        rows = list(csv.reader(io.StringIO(out)))
        h = rows[0]
        ix = {k: i for i, k in enumerate(h)}
        tu = rows[1][ix["gpu__time_duration.sum"]]
        for row in rows[2:]:
            def g(k):
                try:
                    return float(row[ix[k]])
                except (KeyError, ValueError):
                    return float("nan")
            dmma = g("SM_C.TriageCompute.smsp__pipe_tensor_subpipe_dmma_cycles_active.avg")
            el = g("sm__cycles_elapsed.avg")
            st = sorted(((g(k), k.split("issue_stalled_")[1].split("_per_issue")[0]) for k in h
                         if k.startswith("smsp__average_warps_issue_stalled_") and k.endswith("per_issue_active.ratio")),
                        reverse=True)[:4]
            print(f"{row[ix['Kernel Name']][:70]:70s} {g('gpu__time_duration.sum'):9.1f} {tu:2s}  grid {row[ix['launch__grid_size']]:>6s}"
                  f"  DMMA {100 * dmma / el:5.1f} %  warps {g('sm__warps_active.avg.pct_of_peak_sustained_active'):5.1f} %"
                  f"  issue {g('smsp__issue_active.avg.pct_of_peak_sustained_active'):5.1f} %  stalls "
                  + ", ".join(f"{n} {v:.2f}" for v, n in st))


if __name__ == "__main__":
    main(sys.argv[1:])
