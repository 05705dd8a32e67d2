#!/bin/bash
export DT_TIMEOUT_MS=10000
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; tail -2 gpurun_out/pytest_gpu.log
grep -E "passed|failed" gpurun_out/pytest_gpu.log | tail -1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k c5b_1g --durations=3 > gpurun_out/pytest_c5b1g.log 2>&1; tail -5 gpurun_out/pytest_c5b1g.log
LAT_SIZES=4,64,256,1024 LAT_CFGS=1024:0 timeout 200 python tools/msg_latency.py
rm -f /tmp/tr.txt
RING_N=4096 RING_C=1048576 RING_D=0 RING_UNIT=V16 RING_REPS=3 DT_XFER_TRACE=/tmp/tr.txt timeout 60 python tools/ring_one.py > /dev/null
cp /tmp/tr.txt gpurun_out/tr_4096_s.txt
