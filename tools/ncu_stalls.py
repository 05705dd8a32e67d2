#!/usr/bin/env python
"""Kernel-level stall breakdown (pc sampling) + instruction/occupancy/DRAM counters
from an ncu --set full report.  Usage: ncu_stalls.py report.ncu-rep [launch index]"""
import csv
import io
import subprocess
import sys

KEYS = ("smsp__inst_executed.sum", "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "sm__warps_active.avg.per_cycle_active", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "l1tex__t_requests_pipe_lsu_mem_local_op_ld.sum")


def main():
    rep = sys.argv[1]
    idx = int(sys.argv[2]) if len(sys.argv) > 2 else 0
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    h, v = rows[0], rows[2 + idx]
    d = dict(zip(h, v))
    print(d.get("Kernel Name", "?"))
    for k in KEYS:
        if k in d:
            print(f"  {k:55s} {d[k]}")
    st = {k.split("stalled_")[1]: float(x.replace(",", "")) for k, x in d.items()
          if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued")}
    tot = sum(st.values()) or 1.0
    for k, x in sorted(st.items(), key=lambda t: -t[1])[:8]:
        print(f"  stall {k:30s} {100 * x / tot:5.1f}%")


if __name__ == "__main__":
    main()
