"""Summarise a DT_XFER_TRACE dump (per-piece globaltimer stamps of the first CTAs of
each op: t0 wait start, t1 flag acquired, t2 piece copied, t3 flag released).
Usage: python tools/xfer_trace.py trace.txt"""
import sys
from collections import defaultdict

import numpy as np


def main():
    rows = [ln.split() for ln in open(sys.argv[1]) if ln.strip() and not ln.startswith("#")]
    by = defaultdict(list)
    stamps = {}
    for r in rows:
        op, role, j, p, *t = map(int, r)
        t = t[:4] if len(t) < 6 else t
        if p == 63:  # kernel-level stamps: entry, setup done, handshake done, control loop done
            stamps[(op, role, j)] = t
            continue
        by[(op, role, j)].append((p, t))
    base = min([t[0] for v in by.values() for _, t in v] + [t[0] for t in stamps.values() if t[0]])
    for key, t in sorted(stamps.items()):
        print(f"op {key[0]} {'send' if key[1] == 0 else 'recv'} cta {key[2]}: entry {(t[0] - base) / 1e3:6.2f} "
              f"setup {(t[1] - base) / 1e3:6.2f} handshake {(t[2] - base) / 1e3:6.2f} "
              f"end {(t[3] - base) / 1e3 if t[3] else float('nan'):6.2f} us")
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
