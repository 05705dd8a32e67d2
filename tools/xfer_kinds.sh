#!/bin/bash
# C3 / C5 / C5b loopback exchange by pipeline kernel family (DT_XFER_KIND), auto depth,
# and a trace of one small message (kernel-level stamps).
export DT_TIMEOUT_MS=5000
S='import json,sys; d=json.loads(sys.stdin.read()); print([(r["chunk"]>>10,r["depth"],r["gbs_per_rank"]) for r in d["config"]["sweep"]])'
for w in c3 c5 c5b; do
  for k in "" 1 2 4; do
    echo "== $w kind=${k:-auto}"
    DT_XFER_KIND=$k timeout 300 python bench.py --workload xfer --xfer-workload $w --xfer-chunks-kib 64,256,1024,4096 \
      --xfer-depths 0 --steps 10 --warmup 3 2>&1 | tail -1 | python -c "$S"
  done
done
rm -f /tmp/tr.txt; RING_N=65536 RING_C=1048576 RING_D=0 RING_UNIT=V16 RING_REPS=3 DT_XFER_TRACE=/tmp/tr.txt timeout 60 python tools/ring_one.py
python tools/xfer_trace.py /tmp/tr.txt | tail -12
