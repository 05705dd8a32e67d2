export DT_TIMEOUT_MS=10000
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "flatten or pipelined" > gpurun_out/t_flat.log 2>&1; tail -5 gpurun_out/t_flat.log
for m in gpu host; do FU_MODE=$m FU_CONFIGS=C5b_1G,C5b_1G timeout 300 python tools/first_use.py; done > gpurun_out/fu.txt 2>&1; cat gpurun_out/fu.txt
{
PROBE_TAG=base timeout 100 python tools/halo_probe.py
PROBE_TAG=kind1 DT_XFER_KIND=1 timeout 100 python tools/halo_probe.py
PROBE_TAG=ctas128 DT_XFER_CTAS=128 timeout 100 python tools/halo_probe.py
PROBE_TAG=piece8k DT_XFER_PIECE=8192 timeout 100 python tools/halo_probe.py
PROBE_TAG=piece128k DT_XFER_PIECE=131072 timeout 100 python tools/halo_probe.py
PROBE_TAG=c256k PROBE_CHUNK=262144 timeout 100 python tools/halo_probe.py
PROBE_TAG=c4m PROBE_CHUNK=4194304 timeout 100 python tools/halo_probe.py
} > gpurun_out/xprobe.txt 2>&1; cat gpurun_out/xprobe.txt
