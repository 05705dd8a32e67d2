mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_xfer.py -m gpu -x -q > gpurun_out/pytest_xfer.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_xfer.log
tail -3 gpurun_out/pytest_xfer.log
for w in c3 c5 c5b; do timeout 300 python bench.py --workload xfer --xfer-workload $w --xfer-chunks-kib 64,256,1024,4096,16384 --xfer-depths 2,4 --steps 10 --warmup 3 2>/dev/null | grep "^{" | python -c "
import sys,json; d=json.loads(sys.stdin.read()); print('$w', [(r['chunk']>>10, r['depth'], r['gbs_per_rank']) for r in d['config']['sweep']], d['config']['spot_parity'])"; done
DT_BENCH_SHARE_GPU=1 timeout 300 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 5 --warmup 3 --no-cpu 2>/dev/null | grep "^{" | python -c "
import sys,json; d=json.loads(sys.stdin.read()); print('2-rank shared-GPU bench', d['value'], json.dumps(d.get('transfer'))[:300])"
DT_BENCH_SHARE_GPU=1 timeout 300 python -m torch.distributed.run --nnodes=1 --nproc-per-node 8 --master-addr 127.0.0.1 --master-port 29534 bench.py --gpus 8 --workload halo --steps 3 --warmup 3 --ring-loopback 2>&1 | grep "^{" | cut -c1-300
