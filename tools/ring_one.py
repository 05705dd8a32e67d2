"""Diagnostic for ncu: a few 64 KiB BYTE messages through the ring (loopback) at 4 MiB fragments."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_hpdc_wubvjd16_b200 import dt  # noqa: E402

b = dt.Type.basic("BYTE").commit()
src = torch.empty(1 << 20, dtype=torch.uint8, device="cuda").random_(0, 255)
dst = torch.zeros_like(src)
comm = dt.Comm(0, 1, 0, chunk_bytes=4 << 20, depth=2, ring_loopback=True)
for _ in range(3):
    comm.sendrecv(src, 64 << 10, b, 0, dst, 64 << 10, b, 0)
torch.cuda.synchronize()
comm.check()
assert torch.equal(dst[:64 << 10], src[:64 << 10])
print("ok")
