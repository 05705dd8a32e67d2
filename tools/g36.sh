# A/B: session-2 library vs current on the halo ring loopback and C3 xfer (same box, same run)
L=paper_conf_hpdc_wubvjd16_b200/lib
for v in s2 s3 s2 s3; do cp $L/libdt_$v.so $L/libdt.so; timeout 300 python bench.py --workload halo --steps 20 --warmup 3 --ring-loopback 2>&1 | grep "^{" | python -c "
import sys,json; d=json.loads(sys.stdin.read()); print('$v halo ring loopback ms', d['ms_per_step'])"; done
cp $L/libdt_s3.so $L/libdt.so
