#!/bin/bash
# message latency under transfer-kernel flag variants (bit 1: no __nanosleep in polls)
export DT_TIMEOUT_MS=10000
mkdir -p gpurun_out
for f in 0 2; do
  echo "flags=$f $(DT_XFER_FLAGS=$f LAT_SIZES=4,64,1024 LAT_CFGS=1024:0 timeout 200 python tools/msg_latency.py 2>&1 | tail -2 | tr '\n' ' ')"
done
rm -f /tmp/tr.txt
RING_N=4096 RING_C=1048576 RING_D=0 RING_UNIT=V16 RING_REPS=3 DT_XFER_FLAGS=2 DT_XFER_TRACE=/tmp/tr.txt timeout 60 python tools/ring_one.py > /dev/null
cp /tmp/tr.txt gpurun_out/tr_4096_f2.txt
