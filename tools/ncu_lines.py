#!/usr/bin/env python
"""Top source lines by warp-stall samples from an ncu report (needs -lineinfo +
--import-source on).  Usage: ncu_lines.py report.ncu-rep [N]"""
import csv
import io
import subprocess
import sys


def main():
    rep = sys.argv[1]
    n = int(sys.argv[2]) if len(sys.argv) > 2 else 25
    raw = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    cur, hdr, agg = None, None, {}
    for r in csv.reader(io.StringIO(raw)):
        if not r:
            continue
        if r[0] == "File Path":
            cur = r[1].split("/")[-1]
            hdr = None
            continue
        if r[0] == "Line No":
            hdr = r
            continue
        if hdr is None or len(r) < 5:
            continue
        try:
            s = float(r[4] or 0)
        except ValueError:
            continue
        key = (cur, r[0], r[1].strip()[:90])
        agg[key] = agg.get(key, 0.0) + s
    tot = sum(agg.values()) or 1.0
    for (f, line, src), s in sorted(agg.items(), key=lambda x: -x[1])[:n]:
        print(f"{100 * s / tot:5.1f}%  {f}:{line}  {src}")


if __name__ == "__main__":
    main()
