mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "host" > gpurun_out/pytest_host.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_host.log
tail -3 gpurun_out/pytest_host.log
python tools/host_probe.py
for v in 1 0; do DT_HOST_PIPE=$v timeout 600 python bench.py --no-cpu --steps 50 2>/dev/null | grep "^{" | python -c "
import sys,json; d=json.loads(sys.stdin.read()); print('pipe=$v', d['value'], d['e2e']['value'], d['e2e']['of_host_link_ceiling'])"; done
