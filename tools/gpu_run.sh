#!/bin/bash
# Parametrised GPU pass (run under gpurun from the repo root):
#   tools/gpu_run.sh [tests] [smoke] [bench] [launches] [ncu=<kernel-regex>] [cmd=<shell command>] ...
# Each step writes its log under gpurun_out/; steps run in the order given.
mkdir -p gpurun_out
nvidia-smi -L > gpurun_out/gpu.txt 2>&1
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
    cmd=*) bash -c "${step#cmd=}" ;;
  esac
done
