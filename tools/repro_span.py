import os, sys
sys.path.insert(0, '/root/repo')
os.environ["DT_FORCE_KERNEL"] = "7"
import numpy as np, torch
import oracle
from paper_conf_hpdc_wubvjd16_b200 import dt
from tools.kind_probe import unsorted_structs
for n in (64, 4096):
    rec, org, parent = unsorted_structs(n)
    t = dt.from_recipe(rec).commit()
    print("form", n, t.plan(1, 0x10000, 0x20000, 0, t.size), flush=True)
    src_h = np.random.default_rng(1).integers(0, 255, parent, dtype=np.uint8)
    src = torch.from_numpy(src_h).cuda()
    pk = torch.empty(t.size, dtype=torch.uint8, device="cuda")
    dt.pack(t, 1, src, pk, origin_offset=org)
    torch.cuda.synchronize()
    exp = oracle.pack(oracle.from_recipe(rec), 1, src_h, org)
    print(n, "pack ok" if np.array_equal(pk.cpu().numpy(), exp) else "PACK MISMATCH", flush=True)
