#!/bin/bash
# Round-2 evidence pass (one B200): GPU tests, smoke, the default bench line, its
# launch list and a full ncu capture of the C2 kernels, the transfer sweeps and
# their ncu capture.  Everything lands in gpurun_out/r02_*.
mkdir -p gpurun_out
export DT_TIMEOUT_MS=10000
bash tools/gpu_run.sh tests smoke bench launches ncu=k_seg
cp gpurun_out/bench.json gpurun_out/r02_bench.json
S='import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps([(r["chunk"]>>10,r["depth"],r["gbs_per_rank"]) for r in d["config"]["sweep"]]), d["config"].get("fused_loopback_gbs_per_rank"))'
{
for w in c3 c5 c5b; do
  echo "== xfer $w p2p"
  timeout 300 python bench.py --workload xfer --xfer-workload $w --xfer-chunks-kib 64,256,1024,4096 --xfer-depths 2,4,0 --steps 10 --warmup 3 2>&1 | tail -1 | python -c "$S"
done
echo "== xfer c3 nccl"; timeout 300 python bench.py --workload xfer --xfer-mode nccl --xfer-chunks-kib 1024,4096 --xfer-depths 2,4 --steps 10 --warmup 3 2>&1 | tail -1 | python -c "$S"
echo "== xfer c3 direct"; timeout 300 python bench.py --workload xfer --xfer-mode direct --steps 10 --warmup 3 2>&1 | tail -1 | python -c "$S"
for m in p2p direct; do for c in 1024 256; do
  echo "== halo $m chunk ${c}K"
  timeout 200 python bench.py --workload halo --xfer-mode $m --xfer-chunks-kib $c --steps 20 --warmup 3 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['config']['us_per_exchange'], d['config']['periodic_self_check'])"
done; done
echo "== halo probe"; timeout 200 python tools/halo_probe.py
echo "== message latency"; LAT_SIZES=4,64,256,1024 LAT_CFGS=1024:0,64:0 timeout 200 python tools/msg_latency.py
echo "== ring probe"; PROBE_CFGS=1024:0,4096:2,256:4,64:0 PROBE_UNIT=V16 timeout 200 python tools/ring_probe.py
} > gpurun_out/r02_xfer.txt 2>&1
RING_N=134217728 RING_C=1048576 RING_D=0 RING_UNIT=V16 RING_REPS=2 timeout 600 ncu --set full --import-source on \
  --clock-control none -k regex:k_xfer -s 1 -c 1 -o gpurun_out/r02_xfer_ncu -f python tools/ring_one.py > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02_xfer_launches.csv \
  python bench.py --workload xfer --xfer-chunks-kib 1024 --xfer-depths 0 --steps 5 --warmup 3 > /dev/null 2>&1
tail -3 gpurun_out/pytest_gpu.log; tail -1 gpurun_out/smoke.log; cat gpurun_out/r02_xfer.txt | head -40
