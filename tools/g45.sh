#!/bin/bash
# session 4: C4 halo ring/hybrid vs CTAs per direction
mkdir -p gpurun_out
for c in 16 32 64 128; do for m in "p2p --ring-loopback" "hybrid --ring-loopback"; do
  echo "== $m ctas=$c" >> gpurun_out/g45_halo.log
  timeout 300 python bench.py --workload halo --xfer-mode $m --xfer-ctas $c --steps 100 --warmup 5 2>&1 | python -c "import sys,json; l=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(l['config']['us_per_exchange'])" >> gpurun_out/g45_halo.log 2>&1
done; done
cat gpurun_out/g45_halo.log
