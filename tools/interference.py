"""f3 (the paper's §5.3/§5.4 minimal-resources study [L22:c1013],
[L22:c1172]): how much a pack/unpack or a pipelined exchange slows a co-running
compute kernel, and how much it is slowed by it, as a function of the SMs the
datatype engine may use.

Co-runner: a chain of bf16 GEMMs (torch.matmul -> cuBLAS; library code is fine
for the co-runner, it is not the hot path) on stream A.  Datatype work on stream
B, looped until the GEMM chain finishes: C2 pack+unpack with DT_MAX_SMS in
{8, 16, 32, 148}, or the C3 loopback ring exchange with DT_XFER_CTAS in
{8, 16, 32, 64}.  Stream B at normal or high priority.  Prints one JSON line per
point: GEMM TFLOP/s alone and co-running, datatype GB/s alone and co-running.
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_hpdc_wubvjd16_b200 import dt  # noqa: E402
from workloads import c2_lower_triangle, c3_block_cyclic  # noqa: E402


def main():
    dev = torch.device("cuda")
    M = int(os.environ.get("IF_GEMM", 8192))
    NG = int(os.environ.get("IF_GEMMS", 40))
    a = torch.randn(M, M, device=dev, dtype=torch.bfloat16)
    b = torch.randn(M, M, device=dev, dtype=torch.bfloat16)
    c = torch.empty(M, M, device=dev, dtype=torch.bfloat16)
    flops = 2.0 * M ** 3 * NG
    sA = torch.cuda.Stream()

    def gemms():
        with torch.cuda.stream(sA):
            for _ in range(NG):
                torch.matmul(a, b, out=c)

    def time_gemm_alone():
        for _ in range(2):
            gemms()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(sA)
        gemms()
        e1.record(sA)
        torch.cuda.synchronize()
        return e0.elapsed_time(e1)

    g_alone = time_gemm_alone()
    print(json.dumps({"gemm": f"{NG} x bf16 {M}^3", "gemm_alone_ms": round(g_alone, 3),
                      "gemm_alone_tflops": round(flops / (g_alone * 1e-3) / 1e12, 1)}), flush=True)

    rec2, org2, par2 = c2_lower_triangle(4096)
    t2 = dt.from_recipe(rec2).commit()
    src2 = torch.empty(par2, dtype=torch.uint8, device=dev).random_(0, 255)
    dst2 = torch.empty_like(src2)
    pk2 = torch.empty(t2.size, dtype=torch.uint8, device=dev)
    rec3, org3, par3 = c3_block_cyclic(8192, 64)
    t3 = dt.from_recipe(rec3).commit()
    A3 = torch.empty(par3, dtype=torch.uint8, device=dev).random_(0, 255)
    B3 = torch.empty_like(A3)

    def corun(work, bytes_per_iter, prio):
        sB = torch.cuda.Stream(priority=prio)
        with torch.cuda.stream(sB):  # alone
            for _ in range(3):
                work(sB)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(sB)
            n0 = 20
            for _ in range(n0):
                work(sB)
            e1.record(sB)
            torch.cuda.synchronize()
            w_alone = e0.elapsed_time(e1) / n0
        # co-running: the GEMM chain on A, the datatype loop on B until A is done
        torch.cuda.synchronize()
        g0, g1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        d0 = torch.cuda.Event(enable_timing=True)
        g0.record(sA)
        d0.record(sB)
        gemms()
        g1.record(sA)
        ends = []
        while not g1.query():  # keep <= 3 iterations queued so the loop tracks the GEMM chain
            if len(ends) >= 3:
                ends[-3].synchronize()
            with torch.cuda.stream(sB):
                work(sB)
            e = torch.cuda.Event(enable_timing=True)
            e.record(sB)
            ends.append(e)
        torch.cuda.synchronize()
        g_co = g0.elapsed_time(g1)
        # iterations that completed while the GEMM chain ran
        done = [d0.elapsed_time(e) for e in ends if d0.elapsed_time(e) <= d0.elapsed_time(g1)]
        n = len(done)
        w_co = (done[-1] / n) if n else float("nan")
        return {"gemm_co_ms": round(g_co, 3), "gemm_slowdown": round(g_co / g_alone, 3),
                "dt_alone_us": round(w_alone * 1e3, 1), "dt_co_us": round(w_co * 1e3, 1),
                "dt_alone_gbs": round(bytes_per_iter / (w_alone * 1e-3) / 1e9, 1),
                "dt_co_gbs": round(bytes_per_iter / (w_co * 1e-3) / 1e9, 1), "dt_iters_co": n}

    for prio_name, prio in (("normal", 0), ("high", -1)):
        for sms in (8, 16, 32, 148):
            os.environ["DT_MAX_SMS"] = str(sms)

            def pk(s):
                dt.pack(t2, 1, src2, pk2, origin_offset=org2, stream=s)
                dt.unpack(t2, 1, pk2, dst2, origin_offset=org2, stream=s)
            r = corun(pk, 4 * t2.size, prio)
            r.update({"work": "C2 pack+unpack", "DT_MAX_SMS": sms, "priority": prio_name})
            print(json.dumps(r), flush=True)
        os.environ.pop("DT_MAX_SMS", None)
        for ctas in (8, 16, 32, 64):
            comm = dt.Comm(0, 1, 0, chunk_bytes=1 << 20, depth=0, ctas=ctas, ring_loopback=True)

            def xf(s, comm=comm):
                comm.sendrecv(A3, 1, t3, 0, B3, 1, t3, 0, sbuf_offset=org3, rbuf_offset=org3, stream=s)
            r = corun(xf, t3.size, prio)
            comm.check()
            comm.free()
            r.update({"work": "C3 loopback ring exchange (GB/s per direction)", "ctas_per_direction": ctas,
                      "priority": prio_name})
            print(json.dumps(r), flush=True)


if __name__ == "__main__":
    main()
