mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "record_span or every_kernel or c5 or pos_len or random_tiny" > gpurun_out/pytest_rec.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_rec.log
timeout 600 python tools/kbench.py --configs C5_64M,C5_1G,C5b_64M,C3,C2 > gpurun_out/kb_default.jsonl 2>&1
DT_FORCE_KERNEL=2 timeout 600 python tools/kbench.py --configs C5_64M,C5_1G > gpurun_out/kb_word.jsonl 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_rec -c 2 -o gpurun_out/rec_full -f python tools/kbench.py --configs C5_64M --reps 1 > gpurun_out/ncu_rec.log 2>&1
tail -3 gpurun_out/pytest_rec.log; cat gpurun_out/kb_default.jsonl gpurun_out/kb_word.jsonl
