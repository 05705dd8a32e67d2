#!/bin/bash
# Round-2 session-2 evidence pass (one B200): GPU tests, smoke, the default bench line, its
# launch list and a full ncu capture of the C2 kernels (roofline.traffic), the transfer
# sweeps, halo, message latency, first use, and an ncu capture of the C4 x-face ring kernel.
mkdir -p gpurun_out
export DT_TIMEOUT_MS=10000
bash tools/gpu_run.sh tests smoke bench launches ncu=k_seg
cp gpurun_out/bench.json gpurun_out/s2_bench.json
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
echo "== kernels"; timeout 300 python tools/kbench.py --configs C1,C2,C3,C4x,C4y,C5_64M,C5b_64M,T16K --reps 10 2>&1 | cut -c1-330
echo "== first use"; for m in gpu pipe host; do FU_MODE=$m FU_CONFIGS=C5b_1G timeout 300 python tools/first_use.py; done
} > gpurun_out/s2_xfer.txt 2>&1
HALO_FACES=x-,x+ timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_xfer -s 2 -c 1 \
  -o gpurun_out/s2_xface_ncu -f python tools/halo_trace.py > /dev/null 2>&1
tail -3 gpurun_out/pytest_gpu.log; tail -1 gpurun_out/smoke.log; cat gpurun_out/s2_xfer.txt | head -60
