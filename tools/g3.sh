mkdir -p gpurun_out
for f in 0 32 64; do timeout 300 python tools/kbench.py --configs C5_64M,C5_1G,C2 --l2fetch $f > gpurun_out/kb_l2f$f.jsonl 2>&1; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_blk -c 1 -o gpurun_out/blk_full -f python tools/kbench.py --configs C5b_64M --reps 1 > gpurun_out/ncu_blk.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_rec -s 1 -c 1 -o gpurun_out/recu_full -f python tools/kbench.py --configs C5_64M --reps 1 > gpurun_out/ncu_recu.log 2>&1
head -50 gpurun_out/kb_l2f*.jsonl
