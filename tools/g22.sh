mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_xfer.py -m gpu -x -q -k "block_spans" > gpurun_out/pytest_xs.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_xs.log
tail -5 gpurun_out/pytest_xs.log
