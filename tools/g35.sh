for f in 0 4; do DT_XFER_FLAGS=$f timeout 300 python bench.py --workload halo --steps 20 --warmup 3 --ring-loopback 2>&1 | grep "^{" | python -c "
import sys,json; d=json.loads(sys.stdin.read()); print('flags=$f halo ring loopback ms', d['ms_per_step'])"; done
DT_XFER_REP=1 timeout 300 python bench.py --workload halo --steps 20 --warmup 3 --ring-loopback 2>&1 | grep "^{" | python -c "
import sys,json; d=json.loads(sys.stdin.read()); print('rep=1 halo ring loopback ms', d['ms_per_step'])"
