mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_rec -s 4 -c 1 -o gpurun_out/recu_full -f python tools/kbench.py --configs C5_64M --reps 1 > gpurun_out/ncu_recu.log 2>&1
tail -3 gpurun_out/ncu_recu.log
