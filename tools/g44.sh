#!/bin/bash
# session 4: hybrid halo parity + C4 halo at N=1 in every mode (ring, fused loopback group, direct, hybrid)
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_xfer.py -m gpu -q -k "halo" > gpurun_out/g44_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/g44_pytest.log
for m in "p2p --ring-loopback" "p2p" "direct" "hybrid --ring-loopback" "hybrid"; do
  echo "== $m" >> gpurun_out/g44_halo.log
  timeout 300 python bench.py --workload halo --xfer-mode $m --steps 100 --warmup 5 >> gpurun_out/g44_halo.log 2>&1
done
tail -3 gpurun_out/g44_pytest.log; cat gpurun_out/g44_halo.log
