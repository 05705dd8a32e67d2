mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_xfer.py tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/pytest_x2.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_x2.log
tail -3 gpurun_out/pytest_x2.log
for w in c3 c5 c5b; do timeout 300 python bench.py --workload xfer --xfer-workload $w --xfer-chunks-kib 64,256,1024,4096,16384 --steps 10 --warmup 3 2>/dev/null | grep "^{" > gpurun_out/x_$w.json; python -c "
import sys,json; d=json.loads(open('gpurun_out/x_$w.json').read()); print('$w', [(r['chunk']>>10, r['depth'], r['gbs_per_rank']) for r in d['config']['sweep']], d['config']['spot_parity'])"; done
timeout 300 python bench.py --workload halo --steps 20 --warmup 3 --ring-loopback 2>&1 | grep "^{" | cut -c1-260
timeout 300 python bench.py --workload halo --steps 20 --warmup 3 2>&1 | grep "^{" | cut -c1-260
