# transfer pipeline without the per-fragment SC fence: parity (xfer suite) + loopback rates
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_xfer.py -m gpu -x -q > gpurun_out/pytest_xfer.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_xfer.log
tail -3 gpurun_out/pytest_xfer.log
for f in 0 4; do for w in c3 c5 c5b; do DT_XFER_FLAGS=$f timeout 300 python bench.py --workload xfer --xfer-workload $w --xfer-chunks-kib 256,1024,4096,16384 --xfer-depths 4 --steps 10 --warmup 3 2>/dev/null | grep "^{" | python -c "
import sys,json; d=json.loads(sys.stdin.read()); print('flags=$f $w', [(r['chunk']>>10, r['gbs_per_rank']) for r in d['config']['sweep']], d['config']['spot_parity'])"; done; done
DT_BENCH_SHARE_GPU=1 timeout 300 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 5 --warmup 3 --no-cpu 2>/dev/null | grep "^{" | python -c "
import sys,json; d=json.loads(sys.stdin.read()); print('2-rank shared-GPU bench', d['value'], json.dumps(d.get('transfer'))[:400])"
