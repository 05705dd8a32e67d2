mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_xfer.py tests/test_gpu_parity.py -m gpu -x -q -k "direct or record_span or every_kernel or c5 or fused" > gpurun_out/pytest_direct.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_direct.log
timeout 300 python bench.py --workload halo --xfer-mode direct --steps 50 > gpurun_out/halo_direct.json 2>&1
timeout 300 python bench.py --workload halo --steps 50 > gpurun_out/halo_p2p.json 2>&1
timeout 300 python bench.py --workload xfer --xfer-mode direct --steps 10 > gpurun_out/xfer_direct.json 2>&1
export DT_BENCH_SHARE_GPU=1
timeout 300 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29557 bench.py --gpus 2 --workload halo --xfer-mode direct --steps 5 --warmup 3 > gpurun_out/halo_direct2.json 2>&1
tail -15 gpurun_out/pytest_direct.log; cat gpurun_out/halo_direct.json gpurun_out/halo_p2p.json gpurun_out/xfer_direct.json; tail -3 gpurun_out/halo_direct2.json
