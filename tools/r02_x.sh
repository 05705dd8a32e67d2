#!/bin/bash
# x-face staging check: GPU tests, C4 kernels, halo ring and direct transports
export DT_TIMEOUT_MS=10000
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
{
timeout 120 python tools/kbench.py --configs C4x,C4y,C5_64M,C3 --reps 10 2>&1 | cut -c1-330
DT_STAGE_G=8 timeout 120 python tools/kbench.py --configs C4x --reps 10 2>&1 | cut -c1-330
PROBE_TAG=base timeout 100 python tools/halo_probe.py
PROBE_TAG=c256k PROBE_CHUNK=262144 timeout 100 python tools/halo_probe.py
for m in p2p direct; do for c in 1024 256; do
  echo "== halo $m chunk ${c}K"
  timeout 200 python bench.py --workload halo --xfer-mode $m --xfer-chunks-kib $c --steps 20 --warmup 3 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['config']['us_per_exchange'], d['config']['periodic_self_check'])"
done; done
} > gpurun_out/r02_x.txt 2>&1
cat gpurun_out/r02_x.txt
