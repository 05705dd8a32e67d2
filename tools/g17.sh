mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "host" > gpurun_out/pytest_host.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_host.log
timeout 600 python bench.py --steps 50 --no-cpu > gpurun_out/b_zc.json 2>&1
DT_HOST_STAGED=1 timeout 600 python bench.py --steps 50 --no-cpu > gpurun_out/b_st.json 2>&1
tail -3 gpurun_out/pytest_host.log; python -c "
import json
for f in ['gpurun_out/b_zc.json','gpurun_out/b_st.json']:
    l=[x for x in open(f) if x.startswith('{')]
    d=json.loads(l[-1]); print(f, d['value'], d['e2e'])
"
