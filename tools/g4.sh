mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "record_span or every_kernel or c5 or pos_len or random_tiny" > gpurun_out/pytest_rec.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_rec.log
timeout 600 python tools/kbench.py --configs C5_64M,C5_1G,C5b_64M > gpurun_out/kb4.jsonl 2>&1
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"k_rec<true" -c 1 -o gpurun_out/recu_full -f python tools/kbench.py --configs C5_64M --reps 1 > gpurun_out/ncu_recu.log 2>&1
tail -3 gpurun_out/pytest_rec.log; cat gpurun_out/kb4.jsonl; tail -3 gpurun_out/ncu_recu.log
