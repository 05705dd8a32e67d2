"""Diagnostic for ncu: a few contiguous messages through the ring (loopback).
Env: RING_N message bytes (64 KiB), RING_C chunk (4 MiB), RING_D depth (2),
RING_UNIT BYTE|V16 (BYTE), RING_REPS (3)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_hpdc_wubvjd16_b200 import dt  # noqa: E402

n = int(os.environ.get("RING_N", 64 << 10))
unit = os.environ.get("RING_UNIT", "BYTE")
b = dt.Type.basic("BYTE").commit() if unit == "BYTE" else dt.Type.basic("INT64").contiguous(2).commit()
es = 1 if unit == "BYTE" else 16
src = torch.empty(n, dtype=torch.uint8, device="cuda").random_(0, 255)
dst = torch.zeros_like(src)
comm = dt.Comm(0, 1, 0, chunk_bytes=int(os.environ.get("RING_C", 4 << 20)), depth=int(os.environ.get("RING_D", 2)),
               ring_loopback=True)
for _ in range(int(os.environ.get("RING_REPS", 3))):
    comm.sendrecv(src, n // es, b, 0, dst, n // es, b, 0)
torch.cuda.synchronize()
comm.check()
assert torch.equal(dst, src)
print("ok")
