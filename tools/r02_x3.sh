#!/bin/bash
export DT_TIMEOUT_MS=10000
mkdir -p gpurun_out
RING_C=1048576 bash tools/trace_msg.sh "4096 65536"
{
S='import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps([(r["chunk"]>>10,r["depth"],r["gbs_per_rank"]) for r in d["config"]["sweep"]]), d["config"].get("fused_loopback_gbs_per_rank"))'
for w in c3 c5 c5b; do
  echo "== xfer $w p2p"
  timeout 300 python bench.py --workload xfer --xfer-workload $w --xfer-chunks-kib 64,256,1024,4096 --xfer-depths 0 --steps 10 --warmup 3 2>&1 | tail -1 | python -c "$S"
done
PROBE_TAG=base timeout 100 python tools/halo_probe.py
echo "== message latency"; LAT_SIZES=4,64,256,1024 LAT_CFGS=1024:0 timeout 200 python tools/msg_latency.py
echo "== message latency nocoop"; DT_XFER_NOCOOP=1 LAT_SIZES=4,64 LAT_CFGS=1024:0 timeout 200 python tools/msg_latency.py
} > gpurun_out/r02_x3.txt 2>&1
cat gpurun_out/r02_x3.txt
