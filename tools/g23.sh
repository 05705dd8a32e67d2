mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "span" > gpurun_out/pytest_s.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_s.log
for i in 1 2; do timeout 300 python bench.py --workload sweep --sweep C5b_64M --no-cpu 2>&1 | tail -1; done
tail -2 gpurun_out/pytest_s.log
