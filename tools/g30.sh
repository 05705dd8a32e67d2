# replicated sub-rings (2 CTAs per sub-ring, alternating fragments): parity + loopback rates
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_xfer.py -m gpu -x -q > gpurun_out/pytest_xfer.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_xfer.log
tail -3 gpurun_out/pytest_xfer.log
for r in 2 1; do for w in c3 c5 c5b; do DT_XFER_REP=$r timeout 300 python bench.py --workload xfer --xfer-workload $w --xfer-chunks-kib 64,256,1024,4096,16384 --xfer-depths 2,4 --steps 10 --warmup 3 2>/dev/null | grep "^{" | python -c "
import sys,json; d=json.loads(sys.stdin.read()); print('rep=$r $w', [(r['chunk']>>10, r['depth'], r['gbs_per_rank']) for r in d['config']['sweep']], d['config']['spot_parity'])"; done; done
