mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_xfer.py -m gpu -x -q > gpurun_out/pytest_x3.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_x3.log
tail -2 gpurun_out/pytest_x3.log
timeout 300 python bench.py --workload xfer --xfer-workload c3 --xfer-chunks-kib 64,1024,4096 --xfer-depths 4,8 --steps 10 --warmup 3 2>/dev/null | grep "^{" | python -c "
import sys,json; d=json.loads(sys.stdin.read()); print('c3', [(r['chunk']>>10, r['depth'], r['gbs_per_rank']) for r in d['config']['sweep']], d['config']['spot_parity'])"
timeout 300 python bench.py --workload halo --steps 20 --warmup 3 --ring-loopback 2>&1 | grep "^{" | cut -c1-260
