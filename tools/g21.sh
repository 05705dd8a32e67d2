# session 3: full SURVEY 8(d) sweep with the block-span kernel
mkdir -p gpurun_out
timeout 1500 python bench.py --workload sweep > gpurun_out/sweep_s3.jsonl 2> gpurun_out/sweep_s3.err
tail -3 gpurun_out/sweep_s3.jsonl
