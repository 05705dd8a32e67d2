#!/bin/bash
# Per-piece trace of small contiguous loopback messages (last of RING_REPS launches).
mkdir -p gpurun_out
for n in ${1:-4096 65536}; do
  rm -f /tmp/tr.txt
  RING_N=$n RING_C=${RING_C:-1048576} RING_D=0 RING_UNIT=V16 RING_REPS=3 DT_XFER_TRACE=/tmp/tr.txt timeout 60 python tools/ring_one.py > /dev/null
  cp /tmp/tr.txt gpurun_out/tr_$n.txt
done
