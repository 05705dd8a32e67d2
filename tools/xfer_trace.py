"""Summarise a DT_XFER_TRACE dump (per-piece globaltimer stamps of the first CTAs of
each op: t0 wait start, t1 flag acquired, t2 piece copied, t3 flag released).
Usage: python tools/xfer_trace.py trace.txt"""
import sys
from collections import defaultdict

import numpy as np


def main():
    rows = [ln.split() for ln in open(sys.argv[1]) if ln.strip() and not ln.startswith("#")]
    by = defaultdict(list)
    for r in rows:
        op, role, j, p, *t = map(int, r)
        by[(op, role, j)].append((p, t))
    base = min(t[0] for v in by.values() for _, t in v)
    for (op, role, j), v in sorted(by.items()):
        v.sort()
        t = np.array([x[1] for x in v], dtype=np.float64) - base
        wait = np.median(t[:, 1] - t[:, 0]) / 1e3
        copy = np.median(t[:, 2] - t[:, 1]) / 1e3
        rel = np.median(t[:, 3] - t[:, 2]) / 1e3
        gap = np.median(t[1:, 0] - t[:-1, 3]) / 1e3 if len(t) > 1 else 0
        per = (t[-1, 3] - t[0, 0]) / max(1, len(t)) / 1e3
        print(f"op {op} {'send' if role == 0 else 'recv'} cta {j}: n={len(t)} start {t[0, 0] / 1e3:7.2f} us  "
              f"median wait {wait:6.2f} copy {copy:6.2f} release {rel:6.2f} gap {gap:5.2f}  per piece {per:6.2f} us")
        if j == 0 and op < 2:
            print("   first 6 pieces (us from start):", [tuple(round(x / 1e3, 2) for x in row) for row in t[:6]])


if __name__ == "__main__":
    main()
