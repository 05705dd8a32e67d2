mkdir -p gpurun_out
export DT_BENCH_SHARE_GPU=1
TR="python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29555"
timeout 400 $TR bench.py --gpus 2 --steps 20 --warmup 3 --no-cpu > gpurun_out/b2.json 2> gpurun_out/b2.err; echo "rc=$?" >> gpurun_out/b2.err
timeout 400 $TR bench.py --gpus 2 --workload xfer --steps 5 --warmup 3 --xfer-chunks-kib 1024 --xfer-depths 4 > gpurun_out/b2x.json 2> gpurun_out/b2x.err; echo "rc=$?" >> gpurun_out/b2x.err
timeout 400 python -m torch.distributed.run --nnodes=1 --nproc-per-node 8 --master-addr 127.0.0.1 --master-port 29556 bench.py --gpus 8 --workload halo --steps 10 --warmup 3 > gpurun_out/b8h.json 2> gpurun_out/b8h.err; echo "rc=$?" >> gpurun_out/b8h.err
cat gpurun_out/b2.json gpurun_out/b2x.json gpurun_out/b8h.json; tail -3 gpurun_out/b2.err gpurun_out/b2x.err gpurun_out/b8h.err
