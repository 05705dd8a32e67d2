#!/bin/bash
export DT_TIMEOUT_MS=10000
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
{
timeout 200 python tools/kbench.py --configs C5b_64M,C5b_1M,C2,C5_64M --reps 10 2>&1 | cut -c1-330
PROBE_TAG=base timeout 100 python tools/halo_probe.py
PROBE_TAG=sys DT_XFER_SYS=1 timeout 100 python tools/halo_probe.py
S='import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps([(r["chunk"]>>10,r["depth"],r["gbs_per_rank"]) for r in d["config"]["sweep"]]), d["config"].get("fused_loopback_gbs_per_rank"))'
for w in c3 c5b; do
  echo "== xfer $w p2p"
  timeout 300 python bench.py --workload xfer --xfer-workload $w --xfer-chunks-kib 64,1024,4096 --xfer-depths 0 --steps 10 --warmup 3 2>&1 | tail -1 | python -c "$S"
done
echo "== xfer c3 p2p sys"
DT_XFER_SYS=1 timeout 300 python bench.py --workload xfer --xfer-workload c3 --xfer-chunks-kib 1024,4096 --xfer-depths 0 --steps 10 --warmup 3 2>&1 | tail -1 | python -c "$S"
} > gpurun_out/r02_x5.txt 2>&1
cat gpurun_out/r02_x5.txt
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/halo_launches.csv python tools/halo_probe.py > /dev/null 2>&1
