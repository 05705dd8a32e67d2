import time, torch, os, sys
sys.path.insert(0, "/root/repo")
from paper_conf_hpdc_wubvjd16_b200 import dt
from workloads import c5b_irregular
rec, org, parent = c5b_irregular(1 << 30)
t = dt.from_recipe(rec).commit()
src = torch.empty(parent, dtype=torch.uint8, device="cuda").random_(0, 255)
pk = torch.empty(t.size, dtype=torch.uint8, device="cuda")
torch.cuda.synchronize()
for i in range(4):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    h0 = time.perf_counter(); e0.record(); dt.pack(t, 1, src, pk, origin_offset=org); e1.record(); h1 = time.perf_counter()
    torch.cuda.synchronize(); h2 = time.perf_counter()
    print(i, "host call ms", round((h1-h0)*1e3,2), "gpu ms", round(e0.elapsed_time(e1),2), "wall", round((h2-h0)*1e3,2))
print("plan", t.plan(1, src.data_ptr() + org, pk.data_ptr(), 0, t.size))
f = t.form(); print("nblocks", f.nblocks, "tsize", f.tsize, "gran", f.granularity)
