#!/bin/bash
# programmatic dependent launch of the transfer kernel: parity suite and message latency
export DT_TIMEOUT_MS=10000
mkdir -p gpurun_out
DT_XFER_PDL=1 timeout 900 python -m pytest tests/test_gpu_xfer.py -q -x > gpurun_out/pytest_pdl.log 2>&1; tail -2 gpurun_out/pytest_pdl.log
for p in 0 1; do
  echo "pdl=$p $(DT_XFER_PDL=$p LAT_SIZES=4,64,256,1024 LAT_CFGS=1024:0,64:0 timeout 200 python tools/msg_latency.py 2>&1 | tail -4 | tr '\n' ' ')"
done
echo "halo pdl=1: $(DT_XFER_PDL=1 timeout 100 python tools/halo_probe.py 2>&1 | tail -1)"
S='import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps([(r["chunk"]>>10,r["depth"],r["gbs_per_rank"]) for r in d["config"]["sweep"]]))'
echo "c3 pdl=1: $(DT_XFER_PDL=1 timeout 300 python bench.py --workload xfer --xfer-workload c3 --xfer-chunks-kib 64,1024,4096 --xfer-depths 0 --steps 10 --warmup 3 2>&1 | tail -1 | python -c "$S")"
