"""Trace one C4 halo exchange (12 ops, loopback ring; HALO_FACES=x-,x+ for a subset) with
DT_XFER_TRACE/DEBUG set by the caller."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_hpdc_wubvjd16_b200 import dt  # noqa: E402
from paper_conf_hpdc_wubvjd16_b200.halo import make_plan  # noqa: E402

n, h = 512, 1
L = n + 2 * h
comm = dt.Comm(0, 1, 0, chunk_bytes=int(os.environ.get("PROBE_CHUNK", 1 << 20)), depth=0, ring_loopback=True)
plan = make_plan(0, n, h, (1, 1, 1))
buf = torch.empty(L ** 3 * 4, dtype=torch.uint8, device="cuda")
faces = tuple(os.environ.get("HALO_FACES", "x-,x+,y-,y+,z-,z+").split(","))
for _ in range(3):
    plan.exchange(comm, buf, faces=faces)
torch.cuda.synchronize()
comm.check()
print("ok")
