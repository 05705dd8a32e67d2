#!/bin/bash
# session 4: ring halo probe with host posting time (host-bound check)
mkdir -p gpurun_out
P="timeout 120 python tools/halo_probe.py"
PROBE_TAG=default $P >> gpurun_out/g48.log 2>&1
PROBE_TAG=norec DT_XFER_NOREC=1 $P >> gpurun_out/g48.log 2>&1
PROBE_TAG=force2 DT_FORCE_KERNEL=2 $P >> gpurun_out/g48.log 2>&1
PROBE_TAG=c256k PROBE_CHUNK=262144 PROBE_DEPTH=4 $P >> gpurun_out/g48.log 2>&1
PROBE_TAG=c4m PROBE_CHUNK=4194304 $P >> gpurun_out/g48.log 2>&1
cat gpurun_out/g48.log
