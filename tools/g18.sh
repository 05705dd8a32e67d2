# session 3: copy/read microbenchmark (C2 headroom) + ncu of k_blk on C5b
mkdir -p gpurun_out
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o /tmp/copy_mlp tools/micro/copy_mlp.cu && timeout 120 /tmp/copy_mlp > gpurun_out/copy_mlp.txt 2>&1
timeout 300 python bench.py --workload sweep --sweep C5b_64M --no-cpu > gpurun_out/c5b.jsonl 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_blk -c 2 -o gpurun_out/c5b_full -f python bench.py --workload sweep --sweep C5b_64M --no-cpu > gpurun_out/c5b_ncu.log 2>&1
cat gpurun_out/copy_mlp.txt; tail -3 gpurun_out/c5b.jsonl
