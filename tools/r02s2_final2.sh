#!/bin/bash
# Round-2 session-2 closing pass (one B200): GPU tests, smoke, the default bench line and its
# launch list, halo/transfer/latency re-check with the final library.
mkdir -p gpurun_out
export DT_TIMEOUT_MS=10000
bash tools/gpu_run.sh tests smoke bench launches
cp gpurun_out/bench.json gpurun_out/s2f_bench.json
S='import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps([(r["chunk"]>>10,r["depth"],r["gbs_per_rank"]) for r in d["config"]["sweep"]]), d["config"].get("fused_loopback_gbs_per_rank"))'
{
for w in c3 c5 c5b; do
  echo "== xfer $w p2p"
  timeout 300 python bench.py --workload xfer --xfer-workload $w --xfer-chunks-kib 64,256,1024,4096 --xfer-depths 0 --steps 10 --warmup 3 2>&1 | tail -1 | python -c "$S"
done
for m in p2p direct; do
  echo "== halo $m chunk 1024K"
  timeout 200 python bench.py --workload halo --xfer-mode $m --xfer-chunks-kib 1024 --steps 20 --warmup 3 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['config']['us_per_exchange'], d['config']['periodic_self_check'])"
done
echo "== halo probe"; timeout 200 python tools/halo_probe.py
for p in 0 1; do echo "== message latency pdl=$p"; DT_XFER_PDL=$p LAT_SIZES=4,64,256,1024 LAT_CFGS=1024:0 timeout 200 python tools/msg_latency.py; done
} > gpurun_out/s2f_xfer.txt 2>&1
tail -3 gpurun_out/pytest_gpu.log; tail -1 gpurun_out/smoke.log; cat gpurun_out/s2f_xfer.txt
