#!/usr/bin/env python
"""Benchmark of the hot path: pack + unpack of the paper's lower-triangular
matrix (BASELINE.json configs[1]: 4096x4096 f64 lower triangle via
MPI_Type_indexed, PAPER.md [L22:c2839 §5.1]) on B200, one rank per GPU.

One step = dt_pack of the whole triangle from the column-major matrix into a
contiguous buffer + dt_unpack of it into a second matrix (all §8(a) rows that
run on one GPU: S3 position resolve, S4 work split, S5 pack, S6 unpack; S1/S2
construct + commit happen once, before timing, as the paper's cached DEVs
[L24:c2714]).  Metric (BASELINE.json): pack/unpack GB/s counting payload bytes
read + written, i.e. 2*payload per kernel, reported against the measured HBM
copy peak.  At N>1 the headline is the north_star's multi-GPU metric instead:
the pipelined C3 exchange between pairs (r, r^1) through dt_sendrecv over NVLink
(whole-job bytes received per second; roofline = one rank's GB/s per direction
against 900 GB/s), with the same bytes contiguous through the same path (the
paper's "C" comparator) and through NCCL, the NCCL mode, the direct plan, the C4
halo and C5 pairs in a "transfer" object, and the replicated C2 pack/unpack in a
side field (`--workload xfer` / `halo` sweep them further).

L2 hygiene: a 2xL2 scratch buffer is rewritten before every timed kernel, and
only the pack/unpack kernels themselves are inside the CUDA-event intervals.

`--impl reference` times the CPU oracle (oracle/) on the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "pack/unpack GB/s vs HBM peak; GPU↔GPU non-contig transfer GB/s vs NVLink"
UNIT = "GB/s"
WORKLOAD = "C2: lower triangle of 4096x4096 f64 (MPI_Type_indexed, 4096 blocks of 8..32768 B), pack+unpack"


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d.get("hbm_gbs", 6650.0)), "measured"
    return 6650.0, "fallback"


class ClockSampler:
    """Samples SM clock and clock-event reasons with NVML during the timed region."""

    REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
               0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
               0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting"}

    def __init__(self, index):
        self.samples, self.reasons, self.max_mhz = [], 0, None
        self._stop = threading.Event()
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:  # noqa: BLE001
            self.nv = None

    def _run(self):
        while not self._stop.is_set():
            self.sample()
            time.sleep(0.01)

    def sample(self):
        if self.nv is None:
            return
        try:
            self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
            self.reasons |= self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
        except Exception:  # noqa: BLE001
            pass

    def __enter__(self):
        self.t = threading.Thread(target=self._run, daemon=True)
        self.t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        self.t.join()
        self.sample()

    def summary(self):
        rs = [n for b, n in self.REASONS.items() if self.reasons & b and n != "gpu_idle"]
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None, "sm_max_mhz": self.max_mhz,
                "reasons": rs, "samples": len(self.samples)}


def dist_init():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if ws > 1:
        import torch.distributed as tdist
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        import torch
        # test aid: DT_BENCH_SHARE_GPU=1 maps every rank onto the visible GPUs round-robin
        # (several ranks per GPU talk over CUDA IPC exactly as across GPUs) with a gloo
        # process group for the bootstrap and the max-over-ranks reductions
        if os.environ.get("DT_BENCH_SHARE_GPU") == "1":
            local = local % torch.cuda.device_count()
            torch.cuda.set_device(local)
            tdist.init_process_group("gloo")
        else:
            torch.cuda.set_device(local)
            tdist.init_process_group("nccl", device_id=torch.device("cuda", local))
    return ws, rank, local


def c2_buffers(torch, n=4096):
    from workloads import c2_lower_triangle, fill_bytes, seed_for
    rec, org, parent = c2_lower_triangle(n)
    src_h = fill_bytes(parent, seed_for(2))
    return rec, org, parent, src_h


def time_oracle_c2(seconds=10.0, threads=1):
    """CPU oracle (as it stands) on the C2 workload: pack + unpack per rep."""
    import numpy as np

    import oracle
    from workloads import c2_lower_triangle, fill_bytes, seed_for
    rec, org, parent = c2_lower_triangle(4096)
    ot = oracle.from_recipe(rec)
    src = fill_bytes(parent, seed_for(2))
    dst = np.full(parent, 0xA5, dtype=np.uint8)
    payload = ot.size
    reps, t0 = 0, time.perf_counter()
    tp = tu = 0.0
    while True:
        a = time.perf_counter()
        packed = oracle.pack(ot, 1, src, org, threads=threads)
        b = time.perf_counter()
        oracle.unpack(ot, 1, packed, dst, org, threads=threads)
        c = time.perf_counter()
        tp += b - a
        tu += c - b
        reps += 1
        if c - t0 >= seconds:
            break
    value = 4.0 * payload * reps / (tp + tu) / 1e9
    return {"value": round(value, 4), "unit": UNIT, "cores": threads, "kind": "oracle",
            "sample": f"{reps} x (pack+unpack of the full C2 triangle, {payload} B payload), "
                      f"{tp + tu:.1f} s wall, one process, {threads} thread(s)"}, reps, tp + tu


def _cpu_model():
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


def oracle_c2_steps(steps, warmup, budget_s=90.0, rate=1.7e9):
    """The reference arm: W untimed and K timed steps of the CPU oracle (1 thread) on the
    C2 workload; a step packs and unpacks the stream bytes [0, L) -- the whole triangle
    when K + W steps fit ~budget_s at the oracle's ~rate (R+W bytes/s), else a bounded
    prefix sample of it (position-resumed pack/unpack, the same definition)."""
    import numpy as np

    import oracle
    from workloads import c2_lower_triangle, fill_bytes, seed_for
    rec, org, parent = c2_lower_triangle(4096)
    ot = oracle.from_recipe(rec)
    src = fill_bytes(parent, seed_for(2))
    dst = np.full(parent, 0xA5, dtype=np.uint8)
    payload = ot.size
    frac = min(1.0, budget_s * rate / (max(1, steps + warmup) * 4.0 * payload))
    L = max(8, int(payload * frac) & ~7)
    for _ in range(warmup):
        oracle.unpack(ot, 1, oracle.pack(ot, 1, src, org, 0, L), dst, org)
    t0 = time.perf_counter()
    for _ in range(steps):
        oracle.unpack(ot, 1, oracle.pack(ot, 1, src, org, 0, L), dst, org)
    wall = time.perf_counter() - t0
    value = 4.0 * L * steps / wall / 1e9
    sample = (f"{steps} timed x (pack+unpack of stream bytes [0, {L}) of the C2 triangle, "
              f"{'the whole' if L >= payload else f'{100 * L / payload:.1f} % of the'} {payload} B payload), "
              f"{wall:.1f} s wall, one process, 1 thread")
    return {"value": round(value, 4), "unit": UNIT, "cores": 1, "kind": "oracle", "sample": sample}, wall


def run_reference(args):
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if ws > 1 and rank != 0:
        return
    steps = max(1, args.steps)
    cb, wall = oracle_c2_steps(steps, args.warmup)
    line = {"impl": "reference", "metric": METRIC, "value": cb["value"], "unit": UNIT, "n_gpus": args.gpus,
            "steps": steps, "warmup": args.warmup, "ms_per_step": round(1e3 * wall / steps, 3),
            "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "u8", "data": "synthetic (splitmix64 words)",
            "config": {"workload": WORKLOAD, "impl": "CPU oracle (oracle/oracle.c typemap walk), 1 thread"},
            "cpu_baseline": cb,
            "e2e": {"value": cb["value"], "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def run_ours(args):
    import numpy as np
    import torch

    from paper_conf_hpdc_wubvjd16_b200 import dt
    if int(os.environ.get("WORLD_SIZE", "1")) > 1:
        return run_multi(args)
    ws, rank, local = dist_init()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    rec, org, parent, src_h = c2_buffers(torch)
    t = dt.from_recipe(rec).commit()
    payload = t.size
    src = torch.from_numpy(src_h).to(dev)
    dst = torch.full((parent,), 0xA5, dtype=torch.uint8, device=dev)
    packed = torch.empty(payload, dtype=torch.uint8, device=dev)
    l2 = torch.cuda.get_device_properties(dev).L2_cache_size
    flush = torch.empty(2 * l2, dtype=torch.uint8, device=dev)
    flush_rd = torch.zeros(2 * l2 // 4, dtype=torch.int32, device=dev)

    def l2_flush(v):
        # write a 2xL2 buffer, then read another 2xL2 buffer: the timed kernel starts on
        # a cold L2 that holds no dirty lines of the flush itself
        flush.fill_(v)
        flush_rd.sum()
    s = torch.cuda.current_stream()

    def step(evs=None):
        l2_flush(1)
        if evs: evs[0].record(s)
        dt.pack(t, 1, src, packed, origin_offset=org, stream=s)
        if evs: evs[1].record(s)
        l2_flush(2)
        if evs: evs[2].record(s)
        dt.unpack(t, 1, packed, dst, origin_offset=org, stream=s)
        if evs: evs[3].record(s)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    # correctness spot check of this exact launch configuration against the oracle-free closed form
    M = src_h.view(np.float64).reshape(4096, 4096)
    exp_head = M[np.triu_indices(4096)][:4096].view(np.uint8)
    assert np.array_equal(packed[: exp_head.size].cpu().numpy(), exp_head), "packed stream mismatch"

    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(4)] for _ in range(args.steps)]
    w0, w1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    if ws > 1:
        import torch.distributed as tdist
        tdist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        w0.record(s)
        for i in range(args.steps):
            step(evs[i])
        w1.record(s)
        torch.cuda.synchronize()
    tpk = [e[0].elapsed_time(e[1]) for e in evs]
    tup = [e[2].elapsed_time(e[3]) for e in evs]
    kern_ms = sum(tpk) + sum(tup)
    wall_ms = w0.elapsed_time(w1)
    if ws > 1:
        import torch.distributed as tdist
        x = torch.tensor([kern_ms, wall_ms], dtype=torch.float64, device=dev)
        tdist.all_reduce(x, op=tdist.ReduceOp.MAX)
        kern_ms, wall_ms = float(x[0]), float(x[1])
    bytes_per_step = 4 * payload  # pack R+W + unpack R+W
    value = ws * bytes_per_step * args.steps / (kern_ms * 1e-3) / 1e9
    peak, peak_src = load_peaks()
    avg_pack = statistics.mean(tpk)
    avg_unpack = statistics.mean(tup)
    dom_ms, dom = (avg_pack, "pack") if avg_pack >= avg_unpack else (avg_unpack, "unpack")
    achieved = 2 * payload / (dom_ms * 1e-3) / 1e9
    traffic, traffic_src = None, None
    tp = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tp):
        tj = json.load(open(tp))
        traffic, traffic_src = tj.get(f"c2_{dom}"), tj.get("_source")
    beyond = _beyond_l2(dev, args) if not args.no_beyond else None
    e2e = run_e2e(args, t, src_h, org, parent, payload, dev) if rank == 0 and not args.no_e2e else None
    line = {"metric": METRIC, "value": round(value, 2), "unit": UNIT, "n_gpus": ws, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(kern_ms / args.steps, 5), "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "u8", "data": "synthetic (splitmix64 words)",
            "config": {"workload": WORKLOAD, "payload_bytes": payload, "bytes_per_step": bytes_per_step,
                       "l2": "flushed before every timed kernel (outside the event intervals): 2xL2 scratch write, then 2xL2 scratch read",
                       "ms_per_step_wall_incl_flush": round(wall_ms / args.steps, 4),
                       "pack_ms": round(avg_pack, 5), "unpack_ms": round(avg_unpack, 5),
                       "pack_gbs": round(2 * payload / (avg_pack * 1e-3) / 1e9, 1),
                       "unpack_gbs": round(2 * payload / (avg_unpack * 1e-3) / 1e9, 1),
                       "parallelism": f"replicas x{ws}" if ws > 1 else "1 GPU"},
            "roofline": {"bound": "hbm", "kernel": f"k_seg<{dom}> (dt_{dom})", "achieved": round(achieved, 1),
                         "peak": peak, "peak_source": peak_src, "unit": "GB/s", "frac": round(achieved / peak, 4),
                         "traffic": traffic, "traffic_source": traffic_src,
                         "algorithmic_bytes_per_launch": 2 * payload},
            "gpu_launches": 2 * args.steps, "clocks": clk.summary(), "e2e": e2e}
    if beyond is not None:
        line["beyond_l2"] = beyond
    if rank == 0 and ws == 1 and not args.no_cpu:
        # the oracle as it stands, on every host core the process may use (its pthread
        # mode splits the stream into equal byte ranges), and single-threaded beside it
        cores = len(os.sched_getaffinity(0))
        cb = time_oracle_c2(seconds=args.cpu_seconds, threads=cores)[0]
        one = time_oracle_c2(seconds=args.cpu_seconds / 2, threads=1)[0]
        cb["single_thread"] = {"value": one["value"], "cores": 1, "sample": one["sample"]}
        cb["cpu_model"] = _cpu_model()
        line["cpu_baseline"] = cb
    if rank == 0:
        print(json.dumps(line), flush=True)
    if ws > 1:
        import torch.distributed as tdist
        tdist.destroy_process_group()


# ------------------------------------------------------------------ N > 1 GPUs
MULTI_WORKLOAD = ("C3: ScaLAPACK 2D block-cyclic submatrix (N=8192 f64, nb=64, owner (0,1)), 128 MiB per "
                  "direction, pairwise exchange (r, r^1) through dt_sendrecv (P2P ring over NVLink)")


def reduce_max(vals, dev=None):
    """Max over ranks of a list of floats (the contract's max-over-ranks timing)."""
    import torch
    import torch.distributed as tdist
    if not tdist.is_initialized() or tdist.get_world_size() == 1:
        return [float(v) for v in vals]
    x = torch.tensor([float(v) for v in vals], dtype=torch.float64, device=dev if dev is not None else "cpu")
    tdist.all_reduce(x, op=tdist.ReduceOp.MAX)
    return [float(v) for v in x.tolist()]


def assemble_multi_line(ws, steps, warmup, payload, ring, sub, clocks=None, e2e=None, replica=None, dtype="u8"):
    """The N>1 JSON line (SURVEY §8(d) multi-GPU metric).  ring: the headline ring
    exchange {"ms": max-over-ranks ms per exchange, "chunk", "depth", "gbs_per_rank"};
    sub: side measurements (contiguous comparator, NCCL mode, direct plan, C4 halo,
    C5 pairs, ...), each already reduced over ranks.  value = bytes received by all
    ranks per second (whole job); the roofline is one rank's per-direction GB/s
    against 900 GB/s of NVLink 5 per direction."""
    per_dir = payload / (ring["ms"] * 1e-3) / 1e9
    line = {"metric": METRIC, "value": round(ws * per_dir, 1), "unit": UNIT, "n_gpus": ws, "steps": steps,
            "warmup": warmup, "ms_per_step": round(ring["ms"], 5), "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": dtype, "data": "synthetic (splitmix64 words)",
            "config": {"workload": MULTI_WORKLOAD, "payload_bytes_per_direction": payload,
                       "pairs": "(r, r^1)", "chunk": ring.get("chunk"), "depth": ring.get("depth"),
                       "gbs_per_direction": round(per_dir, 1), "parallelism": f"pairs x{ws // 2}",
                       "l2": "inputs (512 MiB matrices) larger than L2"},
            "roofline": {"bound": "nvlink", "kernel": "k_xfer (dt_sendrecv, P2P ring)",
                         "achieved": round(per_dir, 1), "peak": 900.0, "peak_source": "NVLink 5 per direction (spec)",
                         "unit": "GB/s", "frac": round(per_dir / 900.0, 4), "traffic": None},
            "gpu_launches": steps, "transfer": sub}
    c = sub.get("contiguous_same_bytes") or {}
    if c.get("gbs_per_direction"):
        line["config"]["of_contiguous"] = round(per_dir / c["gbs_per_direction"], 3)
    if clocks is not None:
        line["clocks"] = clocks
    if e2e is not None:
        line["e2e"] = e2e
    if replica is not None:
        line["replica_pack_unpack"] = replica
    return line


def _guard(fn, *a, **k):
    """Run one side measurement; a failure is recorded, not fatal (the headline stands)."""
    if os.environ.get("DT_BENCH_VERBOSE"):
        print(f"[bench] rank {os.environ.get('RANK')}: {getattr(fn, '__name__', fn)} {a[1:2]}", file=sys.stderr,
              flush=True)
    try:
        return fn(*a, **k)
    except Exception as e:  # noqa: BLE001
        return {"error": f"{type(e).__name__}: {e}"[:300]}


def _torch_nccl_contig(ws, rank, local, payload, steps, warmup):
    """ncclSend/ncclRecv of the same number of contiguous bytes (torch.distributed)."""
    import torch
    import torch.distributed as tdist
    if tdist.get_backend() != "nccl":
        return {"skipped": "process group backend is not nccl"}
    dev = torch.device("cuda", local)
    peer = rank ^ 1 if (rank ^ 1) < ws else rank
    a = torch.empty(payload, dtype=torch.uint8, device=dev).random_(0, 255)
    b = torch.empty_like(a)

    def one():
        ops = [tdist.P2POp(tdist.isend, a, peer), tdist.P2POp(tdist.irecv, b, peer)]
        for r in tdist.batch_isend_irecv(ops):
            r.wait()
    for _ in range(warmup):
        one()
    torch.cuda.synchronize()
    tdist.barrier()
    s = torch.cuda.current_stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    for _ in range(steps):
        one()
    e1.record(s)
    torch.cuda.synchronize()
    ms = reduce_max([e0.elapsed_time(e1) / steps], dev)[0]
    return {"how": "torch.distributed batch_isend_irecv (ncclSend/ncclRecv) of contiguous bytes",
            "ms": round(ms, 4), "gbs_per_direction": round(payload / (ms * 1e-3) / 1e9, 1)}


def _halo(ws, rank, local, mode, steps, warmup, chunk=1 << 20):
    import torch

    from paper_conf_hpdc_wubvjd16_b200 import dt
    from paper_conf_hpdc_wubvjd16_b200.halo import make_plan
    dev = torch.device("cuda", local)
    dims = {1: (1, 1, 1), 2: (1, 1, 2), 4: (1, 2, 2), 8: (2, 2, 2)}.get(ws, (1, 1, ws))
    n, h = 512, 1
    L = n + 2 * h
    plan = make_plan(rank, n, h, dims)
    buf = torch.empty(L * L * L * 4, dtype=torch.uint8, device=dev)
    buf.view(torch.int32).random_(0, 1 << 30)
    comm = dt.Comm.from_process_group(device=local, chunk_bytes=chunk, depth=0)
    s = torch.cuda.current_stream()
    if mode == "direct":
        xp = plan.direct_plan(comm, buf)
        one, check = (lambda: xp.start(s)), xp.check
    else:
        one, check = (lambda: plan.exchange(comm, buf, stream=s)), comm.check
    for _ in range(warmup):
        one()
    torch.cuda.synchronize()
    check()
    torch.distributed.barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    for _ in range(steps):
        one()
    e1.record(s)
    torch.cuda.synchronize()
    check()
    ms = reduce_max([e0.elapsed_time(e1) / steps], dev)[0]
    if mode == "direct":
        xp.free()
    comm.free()
    del buf
    torch.cuda.empty_cache()
    return {"grid": list(dims), "mode": mode, "us_per_exchange": round(ms * 1e3, 2),
            "gbs_per_rank": round(6 * n * n * h * 4 / (ms * 1e-3) / 1e9, 1)}


def _multi_e2e(ws, rank, local, t, org, steps):
    """The headline exchange end to end through the public API with host buffers:
    every step copies the send layout's span from pinned host memory to the device,
    runs dt_sendrecv, and copies the received span back to pinned host memory."""
    import torch

    from paper_conf_hpdc_wubvjd16_b200 import dt
    dev = torch.device("cuda", local)
    peer = rank ^ 1 if (rank ^ 1) < ws else rank
    tlb, text = t.true_extent
    lo, span = org + tlb, org + tlb + text  # the layout's bytes are [origin + true_lb, + true_extent)
    hs = torch.empty(span, dtype=torch.uint8).pin_memory()
    hr = torch.empty(span, dtype=torch.uint8).pin_memory()
    ds = torch.empty(span, dtype=torch.uint8, device=dev)
    dr = torch.empty(span, dtype=torch.uint8, device=dev)
    comm = dt.Comm.from_process_group(device=local, chunk_bytes=4 << 20, depth=0)
    s = torch.cuda.current_stream()

    def one():
        ds[lo:].copy_(hs[lo:], non_blocking=True)
        comm.sendrecv(ds, 1, t, peer, dr, 1, t, peer, sbuf_offset=org, rbuf_offset=org)
        hr[lo:].copy_(dr[lo:], non_blocking=True)
    one()
    torch.cuda.synchronize()
    torch.distributed.barrier()
    t0 = time.perf_counter()
    for _ in range(steps):
        one()
    torch.cuda.synchronize()
    el = reduce_max([time.perf_counter() - t0], None)[0]
    comm.check()
    comm.free()
    payload = t.size
    return {"value": round(ws * payload * steps / el / 1e9, 2), "unit": UNIT,
            "h2d_bytes_per_step": span - lo, "d2h_bytes_per_step": span - lo, "steps": steps,
            "note": "pinned host buffers; per step: H2D of the send layout's span, dt_sendrecv, D2H of the "
                    "received span; wall clock, max over ranks"}


def _replica_c2(local, steps, warmup):
    """Every rank packs + unpacks its own C2 triangle (no data-path collective): the
    1-GPU metric, replicated; min over ranks of the per-rank GB/s."""
    import torch

    from paper_conf_hpdc_wubvjd16_b200 import dt
    dev = torch.device("cuda", local)
    rec, org, parent, src_h = c2_buffers(torch)
    t = dt.from_recipe(rec).commit()
    src = torch.from_numpy(src_h).to(dev)
    dst = torch.empty(parent, dtype=torch.uint8, device=dev)
    pk = torch.empty(t.size, dtype=torch.uint8, device=dev)
    flush = torch.empty(2 * torch.cuda.get_device_properties(dev).L2_cache_size, dtype=torch.uint8, device=dev)
    s = torch.cuda.current_stream()
    tot = 0.0
    for i in range(warmup + steps):
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
        flush.fill_(1)
        ev[0].record(s)
        dt.pack(t, 1, src, pk, origin_offset=org)
        ev[1].record(s)
        flush.fill_(2)
        ev[2].record(s)
        dt.unpack(t, 1, pk, dst, origin_offset=org)
        ev[3].record(s)
        torch.cuda.synchronize()
        if i >= warmup:
            tot += ev[0].elapsed_time(ev[1]) + ev[2].elapsed_time(ev[3])
    ms = reduce_max([tot / steps], dev)[0]
    del src, dst, pk, flush
    torch.cuda.empty_cache()
    return {"workload": WORKLOAD, "ms_per_step": round(ms, 5),
            "gbs_per_rank": round(4 * t.size / (ms * 1e-3) / 1e9, 1), "note": "slowest rank; L2 flushed per kernel"}


def run_multi(args):
    """N > 1: the north_star's multi-GPU metric.  Headline = the pipelined C3
    exchange between pairs (r, r^1) through dt_sendrecv's P2P ring (best of 1 and 4
    MiB fragments, auto depth); beside it, in the same run, the same bytes contiguous
    through the same path (the paper's "C" comparator, [L26:c977 §5.2]) and through
    torch/NCCL, the NCCL mode, the copy-engine mode and the direct plan on C3, the C4 halo (ring and direct)
    and C5 pairs.  Replica C2 pack/unpack moves to a side field."""
    import torch
    os.environ.setdefault("DT_TIMEOUT_MS", "15000")
    ws, rank, local = dist_init()
    dev = torch.device("cuda", local)
    steps = max(3, min(args.steps, 10))
    w = args.warmup
    clk = ClockSampler(local)
    if os.environ.get("DT_BENCH_VERBOSE"):
        print(f"[bench] rank {rank}: ring C3 headline", file=sys.stderr, flush=True)
    with clk:
        ring_res, payload, ok, (t, A, B, org) = xfer_sweep(ws, rank, local, [1 << 20, 4 << 20], [0], "p2p", 0,
                                                          steps, w)
    best = max(ring_res, key=lambda r: r["gbs_per_rank"])
    del A, B
    torch.cuda.empty_cache()
    sub = {"ring_sweep": ring_res, "spot_parity": ok}

    def sweep1(mode, workload, chunks=(4 << 20,), depths=(0,)):
        r, pay, okk, (_, a, b, _) = xfer_sweep(ws, rank, local, list(chunks), list(depths), mode, 0, steps, w,
                                               workload)
        del a, b
        torch.cuda.empty_cache()
        bb = max(r, key=lambda x: x["gbs_per_rank"])
        return {"ms": bb["ms"], "gbs_per_direction": bb["gbs_per_rank"], "chunk": bb["chunk"],
                "depth": bb["depth"], "spot_parity": okk, "payload": pay}
    sub["contiguous_same_bytes"] = _guard(sweep1, "p2p", "ctg", (1 << 20, 4 << 20))
    sub["contiguous_same_bytes"]["how"] = "dt_sendrecv of 128 MiB contiguous bytes, same ring (paper's C)"
    sub["nccl_contiguous"] = _guard(_torch_nccl_contig, ws, rank, local, payload, steps, w)
    sub["nccl_mode_c3"] = _guard(sweep1, "nccl", "c3", (4 << 20,), (4,))
    sub["copy_engine_c3"] = _guard(sweep1, "ce", "c3", (4 << 20,))
    sub["direct_plan_c3"] = _guard(sweep1, "direct", "c3")
    sub["c4_halo_ring"] = _guard(_halo, ws, rank, local, "p2p", steps, w)
    sub["c4_halo_direct"] = _guard(_halo, ws, rank, local, "direct", steps, w)
    c5 = {}
    for m in (1 << 10, 1 << 20, 64 << 20):
        c5[str(m)] = _guard(sweep1, "p2p", f"c5:{m}", (1 << 20,))
    sub["c5_pairs"] = c5
    e2e = _guard(_multi_e2e, ws, rank, local, t, org, steps) if not args.no_e2e else None
    replica = _guard(_replica_c2, local, steps, w)
    line = assemble_multi_line(ws, steps, w, payload, best, sub, clocks=clk.summary(), e2e=e2e, replica=replica)
    if rank == 0:
        print(json.dumps(line), flush=True)
    torch.distributed.destroy_process_group()


def _beyond_l2(dev, args):
    """A long-run point L2 cannot flatter: the lower triangle of a 16384^2 f64 matrix
    (2 GiB matrix, 1 GiB payload, 8x L2), pack + unpack, event-timed per kernel."""
    import torch

    from paper_conf_hpdc_wubvjd16_b200 import dt
    from workloads import c2_lower_triangle
    try:
        rec, org, parent = c2_lower_triangle(16384)
        t = dt.from_recipe(rec).commit()
        src = torch.empty(parent, dtype=torch.uint8, device=dev).random_(0, 255)
        dst = torch.empty(parent, dtype=torch.uint8, device=dev)
        pk = torch.empty(t.size, dtype=torch.uint8, device=dev)
        s = torch.cuda.current_stream()
        for _ in range(2):
            dt.pack(t, 1, src, pk)
            dt.unpack(t, 1, pk, dst)
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
        n = 5
        ev[0].record(s)
        for _ in range(n):
            dt.pack(t, 1, src, pk)
        ev[1].record(s)
        for _ in range(n):
            dt.unpack(t, 1, pk, dst)
        ev[2].record(s)
        torch.cuda.synchronize()
        ok = bool(torch.equal(src[: 16384 * 8], dst[: 16384 * 8]))  # column 0 lies wholly in the triangle
        tp, tu = ev[0].elapsed_time(ev[1]) / n, ev[1].elapsed_time(ev[2]) / n
        peak, _ = load_peaks()
        gp, gu = 2 * t.size / (tp * 1e-3) / 1e9, 2 * t.size / (tu * 1e-3) / 1e9
        del src, dst, pk
        torch.cuda.empty_cache()
        return {"workload": "T16K: lower triangle of 16384x16384 f64 (1 GiB payload, 8x L2)",
                "pack_ms": round(tp, 4), "unpack_ms": round(tu, 4), "pack_gbs": round(gp, 1),
                "unpack_gbs": round(gu, 1), "pack_frac": round(gp / peak, 4), "unpack_frac": round(gu / peak, 4),
                "spot_check": ok}
    except Exception as e:  # noqa: BLE001
        return {"error": f"{type(e).__name__}: {e}"[:200]}


def run_e2e(args, t, src_h, org, parent, payload, dev):
    """Same metric through the public host-buffer C-ABI (dt_pack_host/dt_unpack_host):
    H2D of the layout span + pack + D2H of the packed stream, then H2D of the packed
    stream and the destination span + unpack + D2H of the span."""
    import torch

    from paper_conf_hpdc_wubvjd16_b200 import dt
    src = torch.from_numpy(src_h).pin_memory()
    dst = torch.full((parent,), 0xA5, dtype=torch.uint8).pin_memory()
    pk = torch.empty(payload, dtype=torch.uint8).pin_memory()
    s = torch.cuda.current_stream()
    for _ in range(2):
        dt.pack_host(t, 1, src.data_ptr() + org, pk.data_ptr(), stream=s)
        dt.unpack_host(t, 1, pk.data_ptr(), dst.data_ptr() + org, stream=s)
    steps = max(3, min(args.steps, 20))
    t0 = time.perf_counter()
    for _ in range(steps):
        dt.pack_host(t, 1, src.data_ptr() + org, pk.data_ptr(), stream=s)
        dt.unpack_host(t, 1, pk.data_ptr(), dst.data_ptr() + org, stream=s)
    torch.cuda.synchronize()
    el = time.perf_counter() - t0
    # context: the host link itself -- payload bytes H2D and payload bytes D2H at the same
    # time (pinned cudaMemcpyAsync on two streams), the traffic of one zero-copy kernel
    dbuf = torch.empty(2 * payload, dtype=torch.uint8, device=dev)
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    bi = []
    for r in range(4):
        torch.cuda.synchronize()
        c0 = time.perf_counter()
        with torch.cuda.stream(s1):
            dbuf[:payload].copy_(pk, non_blocking=True)
        with torch.cuda.stream(s2):
            dst[:payload].copy_(dbuf[payload:], non_blocking=True)
        torch.cuda.synchronize()
        if r:
            bi.append(time.perf_counter() - c0)
    del dbuf
    t_bi = min(bi)
    span = t.true_extent[1]
    if os.environ.get("DT_HOST_STAGED"):  # staged: the layout span travels both ways
        h2d, d2h, how = 2 * span + payload, payload + span, "staged through device scratch"
    else:  # pinned buffers: the kernels read/write host memory directly (typemap bytes + packed stream)
        h2d, d2h, how = 2 * payload, 2 * payload, "zero-copy kernels on the pinned host buffers"
    val = 4 * payload * steps / el / 1e9
    ceil = 4 * payload / (2 * t_bi) / 1e9  # a step = two kernels, each moving payload each way
    return {"value": round(val, 3), "unit": UNIT,
            "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h, "steps": steps,
            "host_link_ceiling": round(ceil, 3), "of_host_link_ceiling": round(val / ceil, 3),
            "host_link_note": "ceiling = same R+W basis with each kernel's H2D+D2H bytes moved by pinned "
                              "cudaMemcpyAsync on two concurrent streams (measured in this run)",
            "note": f"host pinned buffers, {how}; wall clock incl. every host<->device byte and syncs"}


def xfer_sweep(ws, rank, local, chunks, depths, mode_name, ctas, steps, warmup, workload="c3"):
    """Pairwise C3 exchange through dt_sendrecv over a chunk x depth sweep (S7).
    Returns (results, payload, spot_parity); every timing is the max over ranks of
    the device time between a barrier-aligned pair of CUDA events."""
    import torch

    from paper_conf_hpdc_wubvjd16_b200 import dt
    from workloads import c3_block_cyclic, c5_particles, c5b_irregular, fill_bytes, seed_for
    dev = torch.device("cuda", local)
    peer = rank ^ 1 if (rank ^ 1) < ws else rank
    if workload.startswith("c5:"):  # C5 particle message of a given size (pairs sweep)
        rec, org, parent = c5_particles(int(workload[3:]))
    elif workload == "ctg":  # the paper's "C" comparator: the same bytes as C3, contiguous
        rec, org, parent = ("contiguous", 128 << 20, ("basic", "BYTE")), 0, 128 << 20
    else:
        rec, org, parent = {"c3": c3_block_cyclic, "c5": lambda: c5_particles(128 << 20),
                            "c5b": lambda: c5b_irregular(128 << 20)}[workload]()
    t = dt.from_recipe(rec).commit()
    payload = t.size
    A = torch.from_numpy(fill_bytes(parent, seed_for(3) + rank)).to(dev)
    B = torch.full((parent,), 0xA5, dtype=torch.uint8, device=dev)
    s = torch.cuda.current_stream()
    mode = {"nccl": dt.XFER_NCCL, "ce": dt.XFER_CE}.get(mode_name, dt.XFER_P2P)
    results = []
    if mode_name == "direct":  # persistent direct plan: chunk and depth do not apply
        chunks, depths = [0], [0]
    for chunk in chunks:
        for depth in depths:
            if ws > 1:
                comm = dt.Comm.from_process_group(device=local, chunk_bytes=chunk, depth=depth, mode=mode, ctas=ctas)
            else:
                nid = dt.Comm.nccl_unique_id() if mode == dt.XFER_NCCL else None
                comm = dt.Comm(0, 1, local, chunk_bytes=chunk, depth=depth, mode=mode, nccl_id=nid,
                               ctas=ctas, ring_loopback=True)  # measure the pipeline itself
            if mode_name == "direct":
                ops = ([(A.data_ptr() + org, 1, t, peer, 0)], [(B.data_ptr() + org, 1, t, peer, 0)])
                xp = dt.XPlan.from_process_group(comm, *ops) if ws > 1 else dt.XPlan.local(comm, *ops)
                one = lambda: xp.start(s)  # noqa: E731
                chk = xp.check
            else:
                one = lambda: comm.sendrecv(A, 1, t, peer, B, 1, t, peer, sbuf_offset=org, rbuf_offset=org)  # noqa
                chk = comm.check
            for _ in range(warmup):
                one()
            torch.cuda.synchronize()
            chk()
            if ws > 1:
                torch.distributed.barrier()
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            for _ in range(steps):
                one()
            e1.record(s)
            torch.cuda.synchronize()
            chk()
            ms = e0.elapsed_time(e1) / steps
            if ws > 1:
                x = torch.tensor([ms], dtype=torch.float64, device=dev)
                torch.distributed.all_reduce(x, op=torch.distributed.ReduceOp.MAX)
                ms = float(x[0])
            results.append({"chunk": chunk, "depth": depth, "ms": round(ms, 4),
                            "gbs_per_rank": round(payload / (ms * 1e-3) / 1e9, 1)})
            if mode_name == "direct":
                xp.free()
            comm.free()
    # parity of the last exchange: the typemap bytes of my B must equal the peer's A's
    # (same layout on both sides; gap bytes of B keep their poison)
    exp = torch.from_numpy(fill_bytes(parent, seed_for(3) + peer)).to(dev)
    pb = torch.empty(payload, dtype=torch.uint8, device=dev)
    pe = torch.empty(payload, dtype=torch.uint8, device=dev)
    dt.pack(t, 1, B, pb, origin_offset=org)
    dt.pack(t, 1, exp, pe, origin_offset=org)
    ok = bool(torch.equal(pb, pe))
    del pb, pe
    return results, payload, ok, (t, A, B, org)


def run_xfer(args):
    """S7: pipelined GPU<->GPU exchange of the C3 block-cyclic submatrix (128 MiB per
    direction, 512-B runs) through dt_sendrecv, chunk/depth sweep ([L18:c4394 §4.1]).
    Pairs (r, r^1) exchange concurrently; at N=1 the rank exchanges with itself
    (loopback, the paper's "1GPU" case [L26:c1686]).  value = bytes received by all
    ranks per second (max-over-ranks device time)."""
    import torch

    from paper_conf_hpdc_wubvjd16_b200 import dt
    ws, rank, local = dist_init()
    torch.cuda.set_device(local)
    steps = max(3, min(args.steps, 20))
    results, payload, ok, (t, A, B, org) = xfer_sweep(
        ws, rank, local, [int(x) << 10 for x in args.xfer_chunks_kib.split(",")],
        [int(x) for x in args.xfer_depths.split(",")], args.xfer_mode, args.xfer_ctas, steps, args.warmup,
        args.xfer_workload)
    s = torch.cuda.current_stream()
    best = max(results, key=lambda r: r["gbs_per_rank"])
    value = ws * payload / (best["ms"] * 1e-3) / 1e9
    fused = None
    if ws == 1:  # f1: the same loopback exchange as one fused datatype -> datatype copy (no ring)
        for _ in range(args.warmup):
            dt.copy(t, 1, A, t, 1, B, src_offset=org, dst_offset=org)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        for _ in range(10):
            dt.copy(t, 1, A, t, 1, B, src_offset=org, dst_offset=org)
        e1.record(s)
        torch.cuda.synchronize()
        fused = round(payload / (e0.elapsed_time(e1) / 10 * 1e-3) / 1e9, 1)
    # loopback through the ring moves 4x payload through HBM (pack R+W, unpack R+W); a direct
    # plan (and the fused copy) moves 2x (read once, written once)
    peak = 900.0 if ws > 1 else load_peaks()[0] / (2 if args.xfer_mode == "direct" else 4)
    line = {"metric": METRIC, "value": round(value, 1), "unit": UNIT, "n_gpus": ws, "steps": steps,
            "warmup": args.warmup, "ms_per_step": best["ms"], "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "u8", "data": "synthetic (splitmix64 words)",
            "config": {"workload": ("C3: ScaLAPACK 2D block-cyclic submatrix (N=8192 f64, nb=64, owner (0,1))"
                                    if args.xfer_workload == "c3" else "C5: 128 MiB of LAMMPS-style particles"
                                    if args.xfer_workload == "c5" else
                                    "C5b: 128 MiB irregular hindexed (4..64-byte blocks, 0..60-byte gaps)")
                                   + f", pairwise exchange, mode={args.xfer_mode}",
                       "payload_bytes": payload, "sweep": results, "spot_parity": ok,
                       "fused_loopback_gbs_per_rank": fused,
                       "pairs": "loopback (1 GPU)" if ws == 1 else "(r, r^1)"},
            "roofline": {"bound": "nvlink" if ws > 1 else "hbm", "achieved": best["gbs_per_rank"],
                         "peak": peak, "unit": "GB/s", "frac": round(best["gbs_per_rank"] / peak, 4),
                         "note": "per-direction NVLink 900 GB/s nominal" if ws > 1 else
                                 "loopback: HBM peak / (2 direct, 4 ring) bytes moved per payload byte"},
            "gpu_launches": steps}
    if rank == 0:
        print(json.dumps(line), flush=True)
    if ws > 1:
        torch.distributed.destroy_process_group()


def run_halo(args):
    """C4: 3D halo exchange of 512^3 f32 per rank (ghost width 1), 6 subarray faces
    per rank to 3 peers on a periodic grid (2x2x2 at N=8; reading A17), all 12
    transfers of one exchange in one dt_group.  At N=1 the domain is periodic on
    itself (every face is a loopback transfer)."""
    import numpy as np
    import torch

    from paper_conf_hpdc_wubvjd16_b200 import dt
    from paper_conf_hpdc_wubvjd16_b200.halo import make_plan
    ws, rank, local = dist_init()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    dims = {1: (1, 1, 1), 2: (1, 1, 2), 4: (1, 2, 2), 8: (2, 2, 2)}.get(ws, (1, 1, ws))
    n, h = 512, 1
    L = n + 2 * h
    plan = make_plan(rank, n, h, dims)
    buf = torch.empty(L * L * L * 4, dtype=torch.uint8, device=dev)
    buf.view(torch.int32).random_(0, 1 << 30)
    mode = dt.XFER_NCCL if args.xfer_mode == "nccl" else dt.XFER_P2P
    kw = dict(chunk_bytes=1 << 20, depth=2, mode=mode, ctas=args.xfer_ctas, ring_loopback=args.ring_loopback)
    comm = dt.Comm.from_process_group(device=local, **kw) if ws > 1 else \
        dt.Comm(0, 1, local, nccl_id=dt.Comm.nccl_unique_id() if mode == dt.XFER_NCCL else None, **kw)
    s = torch.cuda.current_stream()
    if args.xfer_mode == "direct":  # one persistent direct plan: one kernel per exchange
        xp = plan.direct_plan(comm, buf, single_rank=ws == 1)
        exchange = lambda: xp.start(s)  # noqa: E731
        check = xp.check
    elif args.xfer_mode == "hybrid":  # y/z faces direct, x faces through the ring on a side stream
        exchange = plan.hybrid(comm, buf, s, single_rank=ws == 1)
        check = exchange.check
    else:
        exchange = lambda: plan.exchange(comm, buf, stream=s)  # noqa: E731
        check = comm.check
    for _ in range(args.warmup):
        exchange()
    torch.cuda.synchronize()
    check()
    ok = None
    if ws == 1:
        A = buf.view(torch.int32).view(L, L, L)
        ok = bool(torch.equal(A[1:-1, 1:-1, 0], A[1:-1, 1:-1, n]) and torch.equal(A[1:-1, 0, 1:-1], A[1:-1, n, 1:-1])
                  and torch.equal(A[0, 1:-1, 1:-1], A[n, 1:-1, 1:-1]))
    steps = max(5, min(args.steps, 100))
    if ws > 1:
        torch.distributed.barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    for _ in range(steps):
        exchange()
    e1.record(s)
    torch.cuda.synchronize()
    check()
    ms = e0.elapsed_time(e1) / steps
    if ws > 1:
        x = torch.tensor([ms], dtype=torch.float64, device=dev)
        torch.distributed.all_reduce(x, op=torch.distributed.ReduceOp.MAX)
        ms = float(x[0])
    face = n * n * h * 4
    value = ws * 6 * face / (ms * 1e-3) / 1e9
    line = {"metric": METRIC, "value": round(value, 1), "unit": UNIT, "n_gpus": ws, "steps": steps,
            "warmup": args.warmup, "ms_per_step": round(ms, 4), "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "u8", "data": "synthetic (random f32 bit patterns)",
            "config": {"workload": f"C4: 3D halo 512^3 f32 per rank, 6 faces x {face} B, grid {dims}, "
                                   f"mode={args.xfer_mode}", "us_per_exchange": round(ms * 1e3, 2),
                       "periodic_self_check": ok, "np": np.__version__},
            "gpu_launches": steps * (2 if args.xfer_mode == "hybrid" else 1)}
    if rank == 0:
        print(json.dumps(line), flush=True)
    if ws > 1:
        torch.distributed.destroy_process_group()


def sweep_configs(which):
    """The SURVEY §8(d) 1-GPU table: C1 (+ misaligned), C2, C3, C4 faces, the C5
    particle sweep 1 KiB..1 GiB (x4 steps), C5b, the V sweep (lda = 2N, reading A3),
    the T sweep and the stair triangle (reading A4)."""
    import workloads as W
    cf = {"C1": lambda: W.c1_submatrix(), "C1b": lambda: W.c1_submatrix(r0=1, c0=1),
          "C2": lambda: W.c2_lower_triangle(), "C3": lambda: W.c3_block_cyclic(),
          "C4x": lambda: W.c4_face("x-"), "C4y": lambda: W.c4_face("y-"), "C4z": lambda: W.c4_face("z-"),
          "C5b_64M": lambda: W.c5b_irregular(64 << 20), "Tstair8K": lambda: W.stair_triangle(8192, 256)}
    for k in range(11):
        m = 1 << (10 + 2 * k)
        cf[f"C5_{m >> 10}K"] = (lambda m=m: W.c5_particles(m))
    for n in (1024, 2048, 4096, 8192, 16384):
        cf[f"V{n >> 10}K"] = (lambda n=n: W.c1_submatrix(n, 2 * n))
        cf[f"T{n >> 10}K"] = (lambda n=n: W.c2_lower_triangle(n))
    if which == "all":
        return cf
    return {k: cf[k] for k in which.split(",")}


def sector_bytes(t, count=1):
    """32-byte DRAM sectors the layout touches (x 32 B): the read floor of a pack
    (SURVEY §8(d) "sector-aware" fraction).  Host-only flatten of the committed type."""
    import numpy as np
    d, ln = t.flatten(count)
    d, ln = np.asarray(d), np.asarray(ln)
    o = np.argsort(d, kind="stable")
    a, b = d[o] // 32, (d[o] + ln[o] - 1) // 32
    prev = np.maximum.accumulate(np.concatenate([[-1], b[:-1]]))
    a = np.maximum(a, prev + 1)
    return int(np.sum(np.maximum(0, b - a + 1))) * 32


def run_sweep(args):
    """`--workload sweep`: one JSON row per SURVEY §8(d) config on one GPU (not the
    driver's headline line): pack/unpack event-timed after an L2 flush, CUDA-graph
    replay per call (L2-resident) for small payloads, a same-run contiguous copy,
    the sector-aware fraction, and the CPU oracle as it stands (single thread and
    all host cores) on a bounded prefix sample of the same stream."""
    import numpy as np
    import torch

    import oracle
    from paper_conf_hpdc_wubvjd16_b200 import dt
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(0)
    peak = load_peaks()[0]
    l2 = torch.cuda.get_device_properties(dev).L2_cache_size
    flush = torch.empty(2 * l2, dtype=torch.uint8, device=dev)
    flush_rd = torch.zeros(2 * l2 // 4, dtype=torch.int32, device=dev)
    s = torch.cuda.current_stream()
    cores = len(os.sched_getaffinity(0))

    def timeit(fn, reps):
        ts = []
        for i in range(reps + 3):
            flush.fill_(i & 0xFF)
            flush_rd.sum()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            fn()
            e1.record(s)
            torch.cuda.synchronize()
            if i >= 3:
                ts.append(e0.elapsed_time(e1))
        return statistics.median(ts)

    def graph_us(fn, n=1000):
        g, gs = torch.cuda.CUDAGraph(), torch.cuda.Stream()
        fn(gs)  # plans / word tables are created outside the capture
        torch.cuda.synchronize()
        with torch.cuda.graph(g, stream=gs):
            for _ in range(n):
                fn(gs)
        g.replay()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        g.replay()
        e1.record(s)
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) * 1e3 / n

    for name, mk in sweep_configs(args.sweep).items():
        rec, org, parent = mk()
        t = dt.from_recipe(rec)
        c0 = time.perf_counter()
        t.commit()
        commit_ms = (time.perf_counter() - c0) * 1e3
        n = t.size
        src = torch.empty(parent, dtype=torch.uint8, device=dev)
        src.view(-1)[: parent // 4 * 4].view(torch.int32).random_()
        pk = torch.empty(n, dtype=torch.uint8, device=dev)
        dst = torch.full((parent,), 0xA5, dtype=torch.uint8, device=dev)
        a = torch.empty(n, dtype=torch.uint8, device=dev)
        b = torch.empty(n, dtype=torch.uint8, device=dev)
        reps = 20 if n < (256 << 20) else 7
        pack = lambda st=None: dt.pack(t, 1, src, pk, origin_offset=org, stream=st or s)  # noqa: E731
        unpack = lambda st=None: dt.unpack(t, 1, pk, dst, origin_offset=org, stream=st or s)  # noqa: E731
        tp, tu, tc = timeit(pack, reps), timeit(unpack, reps), timeit(lambda: b.copy_(a), reps)
        kind, gran = t.plan(1, src.data_ptr() + org, pk.data_ptr(), 0, n)
        gbs = lambda ms: round(2 * n / (ms * 1e-3) / 1e9, 1)  # noqa: E731
        row = {"config": name, "payload": n, "kernel": kind, "gran": gran, "commit_ms": round(commit_ms, 2),
               "pack_us": round(tp * 1e3, 2), "unpack_us": round(tu * 1e3, 2), "copy_us": round(tc * 1e3, 2),
               "pack_gbs": gbs(tp), "unpack_gbs": gbs(tu), "copy_gbs": gbs(tc),
               "pack_frac_hbm": round(gbs(tp) / peak, 3), "unpack_frac_hbm": round(gbs(tu) / peak, 3),
               "pack_vs_copy": round(tc / tp, 3), "unpack_vs_copy": round(tc / tu, 3)}
        if n <= (4 << 20):  # latency-bound sizes: per-call device time amortised over 1000 graph-replayed calls
            row["graph_pack_us"] = round(graph_us(pack), 3)
            row["graph_unpack_us"] = round(graph_us(unpack), 3)
            row["graph_note"] = "1000 calls in one CUDA graph, L2-resident (no flush)"
        if n <= (1 << 28):
            sb = sector_bytes(t)
            row["sector_read_bytes"] = sb
            row["pack_sector_aware_frac"] = round((sb + n) / (tp * 1e-3) / 1e9 / peak, 3)
        # CPU oracle as it stands, on a prefix of the same stream (bounded ~1 s per leg)
        ot = oracle.from_recipe(rec)
        host = np.empty(parent, dtype=np.uint8)
        host[: min(parent, 1 << 30)] = 0x5A
        for label, th in (("oracle_1t", 1), ("oracle_mt", cores)):
            m = min(n, 1 << 20)
            while True:
                c0 = time.perf_counter()
                out = oracle.pack(ot, 1, host, org, 0, m, threads=th)
                oracle.unpack(ot, 1, out, host, org, 0, threads=th)
                el = time.perf_counter() - c0
                if el > 0.5 or m >= n:
                    break
                m = min(n, 4 * m)
            row[label + "_gbs"] = round(4 * m / el / 1e9, 3)
            row[label + "_sample_bytes"] = m
        row["oracle_cores"] = cores
        print(json.dumps(row), flush=True)
        del src, pk, dst, a, b, host
        torch.cuda.empty_cache()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--workload", default="c2", choices=["c2", "xfer", "halo", "sweep"])
    ap.add_argument("--sweep", default="all", help="--workload sweep: comma-separated config names or 'all'")
    ap.add_argument("--xfer-mode", default="p2p", choices=["p2p", "nccl", "ce", "direct", "hybrid"],
                    help="p2p ring pipeline, NCCL double buffering, a persistent direct plan (dt_xplan), "
                         "or (halo only) hybrid: y/z faces direct, x faces through the ring")
    ap.add_argument("--xfer-workload", default="c3", choices=["c3", "c5", "c5b"])
    ap.add_argument("--xfer-chunks-kib", default="64,256,1024,4096", help="pipeline fragment sizes (reading A15)")
    ap.add_argument("--xfer-depths", default="2,4,8")
    ap.add_argument("--xfer-ctas", type=int, default=0, help="CTAs per direction (0 = library default)")
    ap.add_argument("--ring-loopback", action="store_true", help="halo at N=1: loopback through the ring pipeline")
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    ap.add_argument("--no-e2e", action="store_true",
                    help="skip the host-buffer e2e leg (ncu launch lists of the timed device step)")
    ap.add_argument("--cpu-seconds", type=float, default=10.0)
    ap.add_argument("--no-beyond", action="store_true", help="skip the beyond-L2 T16K sub-measurement")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.impl == "reference":
        run_reference(args)
    elif args.workload == "xfer":
        if args.xfer_mode == "hybrid":
            ap.error("--xfer-mode hybrid applies to --workload halo only")
        run_xfer(args)
    elif args.workload == "halo":
        run_halo(args)
    elif args.workload == "sweep":
        run_sweep(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
