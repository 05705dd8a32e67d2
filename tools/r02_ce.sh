#!/bin/bash
# copy-engine transfer mode: parity and the C3 sweep next to the P2P kernel and NCCL
export DT_TIMEOUT_MS=10000
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_xfer.py -q -x > gpurun_out/pytest_ce.log 2>&1; tail -3 gpurun_out/pytest_ce.log
S='import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps([(r["chunk"]>>10,r["depth"],r["gbs_per_rank"]) for r in d["config"]["sweep"]]))'
for m in ce p2p; do
  echo "== xfer c3 $m: $(timeout 300 python bench.py --workload xfer --xfer-mode $m --xfer-chunks-kib 64,256,1024,4096 --xfer-depths 2,4,0 --steps 10 --warmup 3 2>&1 | tail -1 | python -c "$S")"
done
