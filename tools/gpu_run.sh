#!/bin/bash
# Parametrised GPU pass (run under gpurun from the repo root):
#   tools/gpu_run.sh [tests] [smoke] [bench] [launches] [ncu=<kernel-regex>]
#                    [xfer=<c3|c5|c5b>[:<mode>]] [halo[=<p2p|direct>]] [probe] [latency] [kbench=<configs>]
#                    [multi=<ranks>] [cmd=<shell command>] ...
# Each step writes its log under gpurun_out/; steps run in the order given.  Tuning
# switches travel in the environment (DT_XFER_FLAGS, DT_XFER_PDL, DT_XFER_SYS,
# DT_FORCE_KERNEL, DT_STAGE_G, DT_MAX_SMS, ...).
mkdir -p gpurun_out
export DT_TIMEOUT_MS=${DT_TIMEOUT_MS:-10000}
nvidia-smi -L > gpurun_out/gpu.txt 2>&1
S='import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps([(r["chunk"]>>10,r["depth"],r["gbs_per_rank"]) for r in d["config"]["sweep"]]), d["config"].get("fused_loopback_gbs_per_rank"))'
for step in "$@"; do
  case "$step" in
    tests) timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1
           echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log; tail -3 gpurun_out/pytest_gpu.log ;;
    smoke) timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
           echo "smoke rc=$?" >> gpurun_out/smoke.log; tail -2 gpurun_out/smoke.log ;;
    bench) timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; cat gpurun_out/bench.json ;;
    launches) timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
                --log-file gpurun_out/launches.csv python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e --no-beyond \
                > gpurun_out/b_ncu.log 2>&1 ;;
    ncu=*) k="${step#ncu=}"
           timeout 900 ncu --set full --clock-control none --import-source on -k "regex:$k" -c 2 \
             -o "gpurun_out/full_${k//[^a-zA-Z0-9_]/_}" -f python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e --no-beyond \
             > "gpurun_out/ncu_${k//[^a-zA-Z0-9_]/_}.log" 2>&1 ;;
    xfer=*) a="${step#xfer=}"; w="${a%%:*}"; m="p2p"; [ "$a" != "$w" ] && m="${a#*:}"
            echo "xfer $w $m: $(timeout 300 python bench.py --workload xfer --xfer-workload $w --xfer-mode $m \
              --xfer-chunks-kib ${XFER_CHUNKS:-64,256,1024,4096} --xfer-depths ${XFER_DEPTHS:-0} --steps 10 --warmup 3 \
              2>&1 | tail -1 | python -c "$S")" | tee -a gpurun_out/steps.txt ;;
    halo|halo=*) m="${step#halo}"; m="${m#=}"; m="${m:-p2p}"
            echo "halo $m: $(timeout 200 python bench.py --workload halo --xfer-mode $m --xfer-chunks-kib 1024 --steps 20 \
              --warmup 3 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['config']['us_per_exchange'], d['config']['periodic_self_check'])")" \
              | tee -a gpurun_out/steps.txt ;;
    probe) echo "halo probe $(timeout 200 python tools/halo_probe.py 2>&1 | tail -1)" | tee -a gpurun_out/steps.txt ;;
    latency) LAT_SIZES=${LAT_SIZES:-4,64,256,1024} LAT_CFGS=${LAT_CFGS:-1024:0} timeout 300 python tools/msg_latency.py \
               2>&1 | tee -a gpurun_out/steps.txt ;;
    kbench=*) timeout 600 python tools/kbench.py --configs "${step#kbench=}" --reps 10 2>&1 | cut -c1-330 \
                | tee -a gpurun_out/steps.txt ;;
    multi=*) n="${step#multi=}"
             DT_BENCH_SHARE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node $n \
               --master-addr 127.0.0.1 --master-port $((29500 + n)) bench.py --gpus $n --steps 3 --warmup 3 \
               > gpurun_out/multi_$n.json 2> gpurun_out/multi_$n.err; echo "multi $n rc=$?" | tee -a gpurun_out/steps.txt ;;
    cmd=*) bash -c "${step#cmd=}" ;;
  esac
done
