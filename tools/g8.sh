mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python tools/kbench.py --configs C1,C1b,C2,C3,C4x,C4y,C4z,C5_64M,C5_1G,C5b_64M,V4K,V8K,V16K,T16K > gpurun_out/kb8.jsonl 2>&1
tail -3 gpurun_out/pytest_gpu.log; cat gpurun_out/kb8.jsonl
