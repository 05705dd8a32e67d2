#!/bin/bash
export DT_TIMEOUT_MS=10000
mkdir -p gpurun_out
{
PROBE_TAG=base timeout 100 python tools/halo_probe.py
for m in p2p direct; do
  echo "== halo $m chunk 1024K"
  timeout 200 python bench.py --workload halo --xfer-mode $m --xfer-chunks-kib 1024 --steps 20 --warmup 3 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['config']['us_per_exchange'], d['config']['periodic_self_check'])"
done
echo "== message latency"; LAT_SIZES=4,64,256,1024 LAT_CFGS=1024:0 timeout 200 python tools/msg_latency.py
} > gpurun_out/r02_x4.txt 2>&1
cat gpurun_out/r02_x4.txt
bash tools/xface_trace.sh
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_span -s 4 -c 2 -o gpurun_out/kspan_full -f python tools/kbench.py --configs C5b_64M --reps 3 > gpurun_out/kspan_ncu.log 2>&1
