"""Print the last launch of a DT_XFER_TRACE dump, times in us from its first stamp."""
import sys

for f in sys.argv[1:]:
    last = open(f).read().split("# launch")[-1].strip().split("\n")[1:]
    rows = [ln.split() for ln in last]
    ts = [int(x) for r in rows for x in r[4:] if int(x)]
    base = min(ts)
    print(f)
    for r in rows:
        op, role, j, p = map(int, r[:4])
        t = [round((int(x) - base) / 1e3, 2) if int(x) else None for x in r[4:]]
        print(" ", "send" if role == 0 else "recv", j, p, t)
