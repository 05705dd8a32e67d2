mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_xfer.py -m gpu -x -q 2>&1 | tail -2
timeout 300 python bench.py --workload sweep --sweep C5b_64M,C5_65536K,C2 --no-cpu 2>/dev/null | grep "^{" | python -c "
import sys,json
for l in sys.stdin:
    d=json.loads(l); print(d['config'], d['kernel'], d['pack_us'], d['unpack_us'])"
