"""Per-message cost of the ring pipeline on one GPU (loopback), separated from host
enqueue cost: a long spin kernel is queued first so that the N messages are all
enqueued before the GPU reaches them; the events around the messages then time the
GPU alone.  Prints host us/call and GPU us/message per (unit, size, chunk).
Env: LAT_SIZES (KiB list), LAT_CFGS (chunkKiB:depth list), LAT_UNITS (BYTE,V16)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_hpdc_wubvjd16_b200 import dt  # noqa: E402


def main():
    sizes = [int(x) << 10 for x in os.environ.get("LAT_SIZES", "4,64,256,1024").split(",")]
    cfgs = [(int(a) << 10, int(b)) for a, b in (x.split(":") for x in os.environ.get("LAT_CFGS", "1024:0,64:0").split(","))]
    units = os.environ.get("LAT_UNITS", "BYTE,V16").split(",")
    src = torch.empty(max(sizes), dtype=torch.uint8, device="cuda").random_(0, 255)
    dst = torch.zeros_like(src)
    s = torch.cuda.Stream()
    torch.cuda.set_stream(s)
    N = 50
    for unit in units:
        b = dt.Type.basic("BYTE").commit() if unit == "BYTE" else dt.Type.basic("INT64").contiguous(2).commit()
        es = 1 if unit == "BYTE" else 16
        for chunk, depth in cfgs:
            comm = dt.Comm(0, 1, 0, chunk_bytes=chunk, depth=depth, ring_loopback=True)
            row = {}
            for n in sizes:
                one = lambda: comm.sendrecv(src, n // es, b, 0, dst, n // es, b, 0, stream=s)  # noqa: E731
                for _ in range(5):
                    one()
                torch.cuda.synchronize()
                torch.cuda._sleep(int(2e7))  # ~10 ms of GPU time: the messages queue up behind it
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s)
                t0 = time.perf_counter()
                for _ in range(N):
                    one()
                host_us = (time.perf_counter() - t0) / N * 1e6
                e1.record(s)
                torch.cuda.synchronize()
                comm.check()
                assert torch.equal(dst[:n], src[:n])
                # the same messages captured once in a CUDA graph and replayed (device-resident
                # sequence numbers): no per-call host work, no per-launch CPU->GPU submission
                g = torch.cuda.CUDAGraph()
                with torch.cuda.graph(g, stream=s):
                    for _ in range(N):
                        one()
                g.replay()
                torch.cuda.synchronize()
                g0, g1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                g0.record(s)
                g.replay()
                g1.record(s)
                torch.cuda.synchronize()
                comm.check()
                row[f"{n >> 10}K"] = (round(e0.elapsed_time(e1) / N * 1e3, 1), round(host_us, 1),
                                      round(g0.elapsed_time(g1) / N * 1e3, 1))
                del g
            print(f"unit={unit} chunk={chunk >> 10}K depth={depth or 'auto'} (gpu us, host us, graph-replay us)/msg:",
                  row, flush=True)
            comm.free()


if __name__ == "__main__":
    main()
