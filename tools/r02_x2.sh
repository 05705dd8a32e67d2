#!/bin/bash
# transfer geometry check: xfer GPU tests, halo ring/direct, message latency, C3 sweep
export DT_TIMEOUT_MS=10000
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_xfer.py -q -x > gpurun_out/pytest_xfer.log 2>&1; tail -3 gpurun_out/pytest_xfer.log
{
PROBE_TAG=base timeout 100 python tools/halo_probe.py
PROBE_TAG=c256k PROBE_CHUNK=262144 timeout 100 python tools/halo_probe.py
for m in p2p direct; do
  echo "== halo $m chunk 1024K"
  timeout 200 python bench.py --workload halo --xfer-mode $m --xfer-chunks-kib 1024 --steps 20 --warmup 3 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['config']['us_per_exchange'], d['config']['periodic_self_check'])"
done
echo "== message latency"; LAT_SIZES=4,64,256,1024 LAT_CFGS=1024:0,64:0 timeout 200 python tools/msg_latency.py
S='import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps([(r["chunk"]>>10,r["depth"],r["gbs_per_rank"]) for r in d["config"]["sweep"]]), d["config"].get("fused_loopback_gbs_per_rank"))'
for w in c3 c5 c5b; do
  echo "== xfer $w p2p"
  timeout 300 python bench.py --workload xfer --xfer-workload $w --xfer-chunks-kib 64,256,1024,4096 --xfer-depths 0 --steps 10 --warmup 3 2>&1 | tail -1 | python -c "$S"
done
} > gpurun_out/r02_x2.txt 2>&1
cat gpurun_out/r02_x2.txt
