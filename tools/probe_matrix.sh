#!/bin/bash
# Transfer-pipeline probe matrix: geometry dump, then 64 MiB / 64 KiB contiguous loopback
# messages under tuning switches (DT_XFER_* env).  Usage: tools/probe_matrix.sh [cfgs]
export PROBE_CFGS="${1:-1024:8,4096:2}"
P="timeout 120 python tools/ring_probe.py"
DT_XFER_DEBUG=1 timeout 60 python - <<'PY' 2>&1 | sort | uniq | head
import torch
from paper_conf_hpdc_wubvjd16_b200 import dt
b=dt.Type.basic("INT64").contiguous(2).commit()
src=torch.zeros(64<<20,dtype=torch.uint8,device="cuda"); dst=torch.zeros_like(src)
for C,D in [(1<<20,8),(4<<20,2),(64<<10,0)]:
    c=dt.Comm(0,1,0,chunk_bytes=C,depth=D,ring_loopback=True)
    c.sendrecv(src,(64<<20)//16,b,0,dst,(64<<20)//16,b,0); torch.cuda.synchronize(); c.free()
PY
for v in "base:" "nosleep:DT_XFER_FLAGS=2" "nofence:DT_XFER_FLAGS=8" "piece128k:DT_XFER_PIECE=131072" "ctas128:DT_XFER_CTAS=128" "ctas16:DT_XFER_CTAS=16" "rep1:DT_XFER_REP=1"; do
  echo "== ${v%%:*}"; env ${v#*:} PROBE_UNIT=V16 $P 2>&1 | tail -2
done
