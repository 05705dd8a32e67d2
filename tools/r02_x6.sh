#!/bin/bash
export DT_TIMEOUT_MS=10000
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_xfer.py tests/test_gpu_parity.py -q -x -k "xfer or loopback or halo or flatten or pipelined or direct" > gpurun_out/pytest_x6.log 2>&1; tail -2 gpurun_out/pytest_x6.log
{
echo "== halo probe"; DT_XFER_DEBUG=1 HALO_FACES=x-,x+ timeout 60 python tools/halo_trace.py 2>&1 | tail -5
timeout 200 python tools/halo_probe.py
for m in p2p direct; do
  echo "== halo $m chunk 1024K"
  timeout 200 python bench.py --workload halo --xfer-mode $m --xfer-chunks-kib 1024 --steps 20 --warmup 3 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['config']['us_per_exchange'], d['config']['periodic_self_check'])"
done
echo "== first use"; for m in gpu gpu pipe; do FU_MODE=$m FU_CONFIGS=C5b_1G,C5b_1G timeout 300 python tools/first_use.py; done
} > gpurun_out/r02_x6.txt 2>&1
cat gpurun_out/r02_x6.txt
