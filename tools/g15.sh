mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_xfer.py -m gpu -x -q > gpurun_out/pytest_xfer.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_xfer.log
timeout 300 python bench.py --workload xfer --xfer-workload c5 --xfer-chunks-kib 1024,4096,16384 --xfer-depths 4 --steps 10 > gpurun_out/x5_rec.json 2>&1
DT_XFER_NOREC=1 timeout 300 python bench.py --workload xfer --xfer-workload c5 --xfer-chunks-kib 1024,4096,16384 --xfer-depths 4 --steps 10 > gpurun_out/x5_norec.json 2>&1
timeout 300 python bench.py --workload xfer --xfer-chunks-kib 1024,4096,16384 --xfer-depths 4 --steps 10 > gpurun_out/x3.json 2>&1
tail -5 gpurun_out/pytest_xfer.log; cat gpurun_out/x5_rec.json gpurun_out/x5_norec.json gpurun_out/x3.json | cut -c1-900
