#!/bin/bash
# copy-group publication (default) vs control-thread publication (DT_XFER_FLAGS=32)
export DT_TIMEOUT_MS=10000
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_xfer.py -q -x > gpurun_out/pytest_grel.log 2>&1; tail -1 gpurun_out/pytest_grel.log
S='import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps([(r["chunk"]>>10,r["depth"],r["gbs_per_rank"]) for r in d["config"]["sweep"]]))'
for f in 0 32; do for sys in 0 1; do
  if [ $sys = 1 ]; then export DT_XFER_SYS=1; else unset DT_XFER_SYS; fi
  echo "flags=$f sys=$sys c3: $(DT_XFER_FLAGS=$f timeout 300 python bench.py --workload xfer --xfer-workload c3 --xfer-chunks-kib 64,256,1024,4096 --xfer-depths 0 --steps 10 --warmup 3 2>&1 | tail -1 | python -c "$S")"
  echo "flags=$f sys=$sys c5b: $(DT_XFER_FLAGS=$f timeout 300 python bench.py --workload xfer --xfer-workload c5b --xfer-chunks-kib 1024,4096 --xfer-depths 0 --steps 10 --warmup 3 2>&1 | tail -1 | python -c "$S")"
  echo "flags=$f sys=$sys halo: $(DT_XFER_FLAGS=$f timeout 100 python tools/halo_probe.py 2>&1 | tail -1)"
done; done
unset DT_XFER_SYS
for f in 0 32; do echo "flags=$f lat: $(DT_XFER_FLAGS=$f LAT_SIZES=4,64,1024 LAT_CFGS=1024:0 timeout 200 python tools/msg_latency.py 2>&1 | tail -1)"; done
