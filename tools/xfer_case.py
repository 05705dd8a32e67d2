"""One loopback ring exchange of a named workload (diagnostics / sanitizer runs).
Usage: python tools/xfer_case.py c3|c5|c5b|v16 [chunk_kib] [depth] [reps]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_hpdc_wubvjd16_b200 import dt  # noqa: E402
from workloads import c3_block_cyclic, c5_particles, c5b_irregular, fill_bytes  # noqa: E402

w = sys.argv[1]
chunk = int(sys.argv[2]) << 10 if len(sys.argv) > 2 else 256 << 10
depth = int(sys.argv[3]) if len(sys.argv) > 3 else 4
reps = int(sys.argv[4]) if len(sys.argv) > 4 else 2
rec, org, parent = {"c3": lambda: c3_block_cyclic(2048, 64), "c5": lambda: c5_particles(3 << 20),
                    "c5b": lambda: c5b_irregular(3 << 20),
                    "v16": lambda: (("contiguous", 1 << 18, ("basic", "INT64")), 0, 2 << 20)}[w]()
t = dt.from_recipe(rec).commit()
A = torch.from_numpy(fill_bytes(parent, 5)).cuda()
B = torch.full((parent,), 0xA5, dtype=torch.uint8, device="cuda")
comm = dt.Comm(0, 1, 0, chunk_bytes=chunk, depth=depth, ring_loopback=True)
for _ in range(reps):
    comm.sendrecv(A, 1, t, 0, B, 1, t, 0, sbuf_offset=org, rbuf_offset=org)
torch.cuda.synchronize()
comm.check()
pa = torch.empty(t.size, dtype=torch.uint8, device="cuda")
pb = torch.empty_like(pa)
dt.pack(t, 1, A, pa, origin_offset=org)
dt.pack(t, 1, B, pb, origin_offset=org)
torch.cuda.synchronize()
print(w, chunk >> 10, depth, "ok" if torch.equal(pa, pb) else "MISMATCH", flush=True)
