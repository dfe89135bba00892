#!/usr/bin/env python
"""Print selected metrics of an ncu report (per kernel launch): `ncu_summary.py report.ncu-rep [regex]`."""
import csv
import io
import re
import subprocess
import sys

KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "dram__bytes.sum.per_second",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active",
    "sm__pipe_tensor_op_dmma_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread", "launch__grid_size",
    "launch__occupancy_limit_registers", "smsp__warps_issue_stalled_barrier_per_warp_active.pct",
    "smsp__warps_issue_stalled_long_scoreboard_per_warp_active.pct",
    "smsp__warps_issue_stalled_short_scoreboard_per_warp_active.pct",
    "smsp__warps_issue_stalled_mio_throttle_per_warp_active.pct",
    "smsp__warps_issue_stalled_math_pipe_throttle_per_warp_active.pct",
    "smsp__warps_issue_stalled_wait_per_warp_active.pct", "smsp__warps_issue_stalled_lg_throttle_per_warp_active.pct",
    "smsp__warps_issue_stalled_not_selected_per_warp_active.pct", "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
]


def main():
    rep = sys.argv[1]
    pat = re.compile(sys.argv[2]) if len(sys.argv) > 2 else None
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h = rows[0]
    ki = h.index("Kernel Name")
    for r in rows[2:]:
        name = r[ki]
        if pat and not pat.search(name):
            continue
        print("==", name[:110])
        for k in KEYS:
            if k in h:
                print(f"   {k:72s} {r[h.index(k)]}")


if __name__ == "__main__":
    main()
