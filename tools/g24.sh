# store-policy experiment: streaming (.cs) vs write-back stores, same box, same run
mkdir -p gpurun_out
L=paper_conf_hpdc_wubvjd16_b200/lib
for v in cs wb cs wb; do cp $L/libdt_$v.so $L/libdt.so; echo "== $v"; timeout 600 python bench.py --workload sweep --sweep C2,C3,C4x,V8K,T8K,C5b_64M,C5_65536K,C5_1048576K --no-cpu 2>/dev/null | python -c "
import sys,json
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); print(d['config'], d['pack_us'], d['unpack_us'], d['copy_us'])
"; done > gpurun_out/storepol.txt 2>&1
cat gpurun_out/storepol.txt
