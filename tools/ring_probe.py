"""Diagnostic: one contiguous message through the ring pipeline on one GPU
(loopback), by message size and fragment size: GPU us per message."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_hpdc_wubvjd16_b200 import dt  # noqa: E402


def main():
    unit = os.environ.get("PROBE_UNIT", "BYTE")  # BYTE: 1-byte granularity; V16: 16-byte elements
    b = dt.Type.basic("BYTE").commit() if unit == "BYTE" else dt.Type.basic("INT64").contiguous(2).commit()
    es = 1 if unit == "BYTE" else 16
    src = torch.empty(64 << 20, dtype=torch.uint8, device="cuda").random_(0, 255)
    dst = torch.zeros_like(src)
    s = torch.cuda.current_stream()
    cfgs = os.environ.get("PROBE_CFGS", "1024:2,1024:0,4096:2,256:4,64:0")
    for chunk, depth in [(int(a) << 10, int(b)) for a, b in (x.split(":") for x in cfgs.split(","))]:
        comm = dt.Comm(0, 1, 0, chunk_bytes=chunk, depth=depth, ring_loopback=True,
                       ctas=int(os.environ.get("PROBE_CTAS", 0)))
        row = {}
        for n in [64 << 10, 256 << 10, 1 << 20, 4 << 20, 16 << 20, 64 << 20]:
            for _ in range(3):
                comm.sendrecv(src, n // es, b, 0, dst, n // es, b, 0, stream=s)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            for _ in range(10):
                comm.sendrecv(src, n // es, b, 0, dst, n // es, b, 0, stream=s)
            e1.record(s)
            torch.cuda.synchronize()
            comm.check()
            assert torch.equal(dst[:n], src[:n])
            row[f"{n >> 10}K"] = round(e0.elapsed_time(e1) / 10 * 1e3, 1)
        print(f"unit={unit} ctas={os.environ.get('PROBE_CTAS', 0)} chunk={chunk >> 10}K depth={depth or 'auto'}", row,
              flush=True)
        comm.free()


if __name__ == "__main__":
    main()
