#!/bin/bash
# Per-piece trace of the C4 x-face exchange through the loopback ring (last of 3 launches).
mkdir -p gpurun_out
for f in "x-,x+" "y-,y+"; do
  rm -f /tmp/tr.txt
  HALO_FACES=$f DT_XFER_DEBUG=1 DT_XFER_TRACE=/tmp/tr.txt timeout 120 python tools/halo_trace.py > gpurun_out/trd_${f//,/_}.txt 2>&1
  cp /tmp/tr.txt gpurun_out/tr_${f//,/_}.txt
done
