#!/usr/bin/env python
"""Top SASS instructions by warp-stall samples from an ncu report (first kernel).
Usage: ncu_sass_top.py report.ncu-rep [min_pct]"""
import csv
import io
import subprocess
import sys


def main():
    rep = sys.argv[1]
    thr = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
    raw = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    h, data = rows[1], []
    for r in rows[2:]:
        if r and r[0] == "Kernel Name":
            break
        data.append(r)
    iS, iE = h.index("Warp Stall Sampling (All Samples)"), h.index("Instructions Executed")
    f = lambda x: float(x) if x not in ("", "-") else 0.0
    tot = sum(f(r[iS]) for r in data) or 1.0
    for i, r in enumerate(data):
        if 100 * f(r[iS]) / tot >= thr:
            print(f"{i:5d} {100 * f(r[iS]) / tot:5.1f}% ex={r[iE]:>8s} {r[1].strip()[:90]}")


if __name__ == "__main__":
    main()
