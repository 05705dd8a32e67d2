mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__cycles_active.max,gpc__cycles_elapsed.max --clock-control none --csv --log-file gpurun_out/c1_launches.csv python tools/kbench.py --configs C1,C4y,C4x --reps 3 > /dev/null 2>&1
python tools/ncu_summary.py launches gpurun_out/c1_launches.csv
