#!/bin/bash
# N>1 bench line on ONE GPU (functional only: ranks time-slice the GPU): 2 and 8 ranks,
# GPU-scope flags and system-scope flags (the cross-GPU configuration's code path)
export DT_TIMEOUT_MS=20000
mkdir -p gpurun_out
for n in 2 8; do for sys in 0 1; do
  echo "== ranks=$n sys=$sys"
  if [ $sys = 1 ]; then export DT_XFER_SYS=1; else unset DT_XFER_SYS; fi
  DT_BENCH_SHARE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node $n --master-addr 127.0.0.1 --master-port $((29500 + n + 10*sys)) bench.py --gpus $n --steps 3 --warmup 3 > gpurun_out/multi_${n}_${sys}.json 2> gpurun_out/multi_${n}_${sys}.err
  echo "rc=$?"; tail -c 1500 gpurun_out/multi_${n}_${sys}.json; echo; grep -i "error\|Traceback" gpurun_out/multi_${n}_${sys}.err | head -5
done; done
