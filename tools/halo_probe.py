"""Diagnostic: C4 halo (512^3 f32, 1 GPU, periodic on itself) through the ring
pipeline (loopback) with the exchange split by face set, event-timed; also the host time spent
posting each exchange (a GPU time equal to it means the loop is host-bound)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_hpdc_wubvjd16_b200 import dt  # noqa: E402
from paper_conf_hpdc_wubvjd16_b200.halo import make_plan  # noqa: E402


def main():
    n, h = 512, 1
    L = n + 2 * h
    chunk = int(os.environ.get("PROBE_CHUNK", 1 << 20))
    depth = int(os.environ.get("PROBE_DEPTH", 0))
    comm = dt.Comm(0, 1, 0, chunk_bytes=chunk, depth=depth, ring_loopback=True)
    plan = make_plan(0, n, h, (1, 1, 1))
    buf = torch.empty(L ** 3 * 4, dtype=torch.uint8, device="cuda")
    buf.view(torch.int32).random_(0, 1 << 30)
    s = torch.cuda.current_stream()
    res = {}
    for name, faces in [("x", ("x-", "x+")), ("y", ("y-", "y+")), ("z", ("z-", "z+")),
                        ("all", ("x-", "x+", "y-", "y+", "z-", "z+"))]:
        for _ in range(3):
            plan.exchange(comm, buf, stream=s, faces=faces)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record(s)
        t0 = time.perf_counter()
        for _ in range(20):
            plan.exchange(comm, buf, stream=s, faces=faces)
        t1 = time.perf_counter()
        e1.record(s)
        torch.cuda.synchronize()
        comm.check()
        # GPU us per exchange, and host us per exchange spent posting it (enqueue only)
        res[name] = (round(e0.elapsed_time(e1) / 20 * 1e3, 1), round((t1 - t0) / 20 * 1e6, 1))
    print(os.environ.get("PROBE_TAG", ""), f"chunk={chunk} depth={depth}", res, flush=True)


if __name__ == "__main__":
    main()
