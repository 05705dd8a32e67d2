mkdir -p gpurun_out
timeout 300 compute-sanitizer --tool memcheck python tools/repro_span.py 2>&1 | tail -4
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_xfer.py -m gpu -x -q -k "span or random or every_kernel or c5b or replicas" 2>&1 | tail -2
python tools/kind_probe.py
