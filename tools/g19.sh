# session 3: block-span kernel (k_span) parity + C5b timing + ncu (pack and unpack)
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "span or every_kernel or c5b" > gpurun_out/pytest_span.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_span.log
timeout 300 python bench.py --workload sweep --sweep C5b_64M --no-cpu > gpurun_out/c5b.jsonl 2>&1
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:k_span<\(bool\)0" -c 1 -o gpurun_out/c5b_span_p -f python bench.py --workload sweep --sweep C5b_64M --no-cpu > gpurun_out/c5b_ncu.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:k_span<\(bool\)1" -c 1 -o gpurun_out/c5b_span_u -f python bench.py --workload sweep --sweep C5b_64M --no-cpu > gpurun_out/c5b_ncu2.log 2>&1
tail -15 gpurun_out/pytest_span.log; tail -2 gpurun_out/c5b.jsonl
