# session 3: block spans inside the ring pipeline (C5b transfers) + xfer regression
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_xfer.py tests/test_gpu_parity.py -m gpu -x -q -k "span or loopback or record" > gpurun_out/pytest_xspan.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_xspan.log
timeout 300 python bench.py --workload xfer --xfer-workload c5b --xfer-chunks-kib 256,1024,4096 --xfer-depths 4 --steps 10 --warmup 3 > gpurun_out/x_c5b.json 2>&1
DT_XFER_NOSPAN=1 timeout 300 python bench.py --workload xfer --xfer-workload c5b --xfer-chunks-kib 1024,4096 --xfer-depths 4 --steps 5 --warmup 2 > gpurun_out/x_c5b_nospan.json 2>&1
timeout 300 python bench.py --workload xfer --xfer-workload c3 --xfer-chunks-kib 1024,4096 --xfer-depths 4 --steps 10 --warmup 3 > gpurun_out/x_c3.json 2>&1
tail -5 gpurun_out/pytest_xspan.log
for f in x_c5b x_c5b_nospan x_c3; do python -c "
import json,sys
l=[x for x in open('gpurun_out/$f.json') if x.startswith('{')]
d=json.loads(l[-1]); print('$f', d['value'], d['config']['sweep'], d['config'].get('spot_parity'))
"; done
