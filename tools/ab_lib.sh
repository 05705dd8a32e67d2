#!/bin/bash
# A/B of library builds on the same box (C3 ring sweep): the tree's libdt.so and the
# ab_*_libdt.so copies placed beside it
export DT_TIMEOUT_MS=10000
S='import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps([(r["chunk"]>>10,r["depth"],r["gbs_per_rank"]) for r in d["config"]["sweep"]]))'
L=paper_conf_hpdc_wubvjd16_b200/lib/libdt.so
cp $L ab_tree_libdt.so
for v in head old head old; do
  cp ab_${v}_libdt.so $L; touch $L
  echo "$v: $(timeout 300 python bench.py --workload xfer --xfer-workload c3 --xfer-chunks-kib 64,1024,4096 --xfer-depths 0 --steps 10 --warmup 3 2>&1 | tail -1 | python -c "$S")"
done
