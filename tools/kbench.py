#!/usr/bin/env python
"""Kernel-level sweep over the paper's workloads (tuning aid, not the driver bench).

For each config: pack and unpack GB/s (payload read + written, 2*size per
kernel) with the L2 flushed before every launch, next to a contiguous device
copy of the same bytes measured in the same run (the paper's "C" / cudaMemcpy
practical-peak comparator, [L22:c3205 §5.1]).  Prints one JSON line per config.
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="C1,C1b,C2,C3,C4x,C4y,C4z,C5_64M,C5_1G,C5b_64M,V4K,V8K,V16K,T16K")
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--l2fetch", type=int, default=0, help="cudaLimitMaxL2FetchGranularity (bytes) for the run")
    ap.add_argument("--naive", default="", help="configs that also time the per-block cudaMemcpyAsync baseline")
    args = ap.parse_args()
    import numpy as np
    import torch

    from paper_conf_hpdc_wubvjd16_b200 import dt
    import workloads as W
    mk = {
        "C1": lambda: W.c1_submatrix(), "C1b": lambda: W.c1_submatrix(r0=1, c0=1),
        "C2": lambda: W.c2_lower_triangle(), "C3": lambda: W.c3_block_cyclic(),
        "C4x": lambda: W.c4_face("x-"), "C4y": lambda: W.c4_face("y-"), "C4z": lambda: W.c4_face("z-"),
        "C5_64M": lambda: W.c5_particles(64 << 20), "C5_1G": lambda: W.c5_particles(1 << 30),
        "C5b_64M": lambda: W.c5b_irregular(64 << 20), "C5b_1G": lambda: W.c5b_irregular(1 << 30),
        "V4K": lambda: W.c1_submatrix(4096, 8192), "V8K": lambda: W.c1_submatrix(8192, 16384),
        "V16K": lambda: W.c1_submatrix(16384, 16384),
        "T16K": lambda: W.c2_lower_triangle(16384), "Tstair8K": lambda: W.stair_triangle(8192, 256),
        "T8K": lambda: W.c2_lower_triangle(8192), "C5b_1M": lambda: W.c5b_irregular(1 << 20),
    }
    dev = torch.device("cuda")
    torch.zeros(1, device=dev)
    if args.l2fetch:
        from cuda.bindings import runtime as cudart
        print(cudart.cudaDeviceSetLimit(cudart.cudaLimit.cudaLimitMaxL2FetchGranularity, args.l2fetch),
              cudart.cudaDeviceGetLimit(cudart.cudaLimit.cudaLimitMaxL2FetchGranularity), file=sys.stderr)
    l2 = torch.cuda.get_device_properties(dev).L2_cache_size
    flush = torch.empty(2 * l2, dtype=torch.uint8, device=dev)
    flush_rd = torch.zeros(2 * l2 // 4, dtype=torch.int32, device=dev)

    def l2_flush(v):
        # write a 2xL2 buffer, then read another 2xL2 buffer: the timed kernel starts on
        # a cold L2 that holds no dirty lines of the flush itself
        flush.fill_(v)
        flush_rd.sum()
    s = torch.cuda.current_stream()
    for name in args.configs.split(","):
        if name.startswith("F8:"):  # Fig. 8 sweep: F8:<nblocks>:<block bytes>, gap = block
            _, nb, bs = name.split(":")
            nb, bs = int(nb), int(bs)
            mk[name] = (lambda nb=nb, bs=bs: (("vector", nb, bs // 8, 2 * bs // 8, ("basic", "DOUBLE")), 0,
                                              2 * bs * nb))
        rec, org, parent = mk[name]()
        t = dt.from_recipe(rec)
        import time as _time
        c0 = _time.perf_counter()
        t.commit()  # f2: first-use cost (host flatten + upload + device scan), cached afterwards
        commit_ms = (_time.perf_counter() - c0) * 1e3
        n = t.size
        src = torch.empty(parent, dtype=torch.uint8, device=dev)
        src.random_(0, 256)
        pk = torch.empty(n, dtype=torch.uint8, device=dev)
        dst = torch.empty(parent, dtype=torch.uint8, device=dev)
        a = torch.empty(n, dtype=torch.uint8, device=dev)
        b = torch.empty(n, dtype=torch.uint8, device=dev)

        def timeit(fn):
            ts = []
            for i in range(args.reps + 3):
                l2_flush(i & 0xFF)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s)
                fn()
                e1.record(s)
                torch.cuda.synchronize()
                if i >= 3:
                    ts.append(e0.elapsed_time(e1))
            return statistics.median(ts)

        tp = timeit(lambda: dt.pack(t, 1, src, pk, origin_offset=org, stream=s))
        tu = timeit(lambda: dt.unpack(t, 1, pk, dst, origin_offset=org, stream=s))
        tc = timeit(lambda: b.copy_(a))
        kind, g = t.plan(1, src.data_ptr() + org, pk.data_ptr(), 0, n)
        gb = lambda ms: round(2 * n / (ms * 1e-3) / 1e9, 1)
        row = {"config": name, "bytes": n, "kernel": kind, "gran": g, "pack_us": round(tp * 1e3, 2),
               "unpack_us": round(tu * 1e3, 2), "copy_us": round(tc * 1e3, 2), "pack_gbs": gb(tp),
               "unpack_gbs": gb(tu), "copy_gbs": gb(tc),
               "pack_vs_copy": round(tc / tp, 3), "unpack_vs_copy": round(tc / tu, 3),
               "commit_ms": round(commit_ms, 3)}
        if rec[0] == "vector" and rec[4][0] == "basic":
            # f4 diagnostic (Fig. 8, [L24:c4075 §5.1]): cudaMemcpy2D of the same vector, device to device
            from cuda.bindings import runtime as cudart
            es = {"DOUBLE": 8, "FLOAT": 4, "INT32": 4}.get(rec[4][1], 8)
            width, height, spitch = rec[2] * es, rec[1], rec[3] * es

            def m2d():
                cudart.cudaMemcpy2DAsync(pk.data_ptr(), width, src.data_ptr() + org, spitch, width, height,
                                         cudart.cudaMemcpyKind.cudaMemcpyDeviceToDevice, s.cuda_stream)
            tm = timeit(m2d)
            row.update({"memcpy2d_us": round(tm * 1e3, 2), "memcpy2d_gbs": gb(tm),
                        "pack_vs_memcpy2d": round(tm / tp, 3)})
        if args.naive and name in args.naive.split(","):
            # f4 naive baseline (Fig. 1c, [L14:c4769 §3]): one device-to-device cudaMemcpyAsync per
            # contiguous block of the flattened typemap -- issued from a host loop (what a user gets),
            # and captured once into a CUDA graph and replayed (the copy engine's per-block floor
            # without host launch cost)
            from cuda.bindings import runtime as cudart
            disp, lens = t.flatten(1)
            offs = np.concatenate([[0], np.cumsum(lens)[:-1]])
            base_s, base_p = src.data_ptr() + org, pk.data_ptr()
            D2D = cudart.cudaMemcpyKind.cudaMemcpyDeviceToDevice

            def loop():
                for d, ln, o in zip(disp.tolist(), lens.tolist(), offs.tolist()):
                    cudart.cudaMemcpyAsync(base_p + o, base_s + d, ln, D2D, s.cuda_stream)
            tl = timeit(loop)
            g = torch.cuda.CUDAGraph()
            cs = torch.cuda.Stream()
            with torch.cuda.stream(cs):
                with torch.cuda.graph(g, stream=cs):
                    for d, ln, o in zip(disp.tolist(), lens.tolist(), offs.tolist()):
                        cudart.cudaMemcpyAsync(base_p + o, base_s + d, ln, D2D, cs.cuda_stream)
            tg = timeit(g.replay)
            dt.pack(t, 1, src, a, origin_offset=org, stream=s)  # the naive copies must build the same stream
            torch.cuda.synchronize()
            row["naive_parity"] = bool(torch.equal(pk, a))
            row.update({"naive_blocks": int(len(lens)), "naive_loop_us": round(tl * 1e3, 1),
                        "naive_loop_gbs": gb(tl), "naive_graph_us": round(tg * 1e3, 1), "naive_graph_gbs": gb(tg),
                        "pack_vs_naive_loop": round(tl / tp, 1), "pack_vs_naive_graph": round(tg / tp, 1)})
            del g
        print(json.dumps(row), flush=True)
        del src, pk, dst, a, b
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
