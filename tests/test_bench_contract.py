"""The driver's bench.py contract on CPU: the --impl reference arm (the CPU oracle
on the C2 workload) prints one JSON line with the required keys, and the
argument parser accepts the driver's launch flags."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_reference_arm_json_line():
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--gpus", "1",
                          "--steps", "1", "--warmup", "3"], capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [ln for ln in out.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
              "vs_baseline", "dtype", "data", "config", "cpu_baseline", "e2e"):
        assert k in d, k
    assert d["impl"] == "reference" and d["value"] > 0 and d["unit"] == "GB/s"
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["value"] == d["value"]
    assert "workload" in d["config"]
    assert (d["steps"], d["warmup"]) == (1, 3)  # exactly the requested K timed / W warm-up steps


def test_reference_arm_nonzero_rank_is_silent():
    env = dict(os.environ, WORLD_SIZE="2", RANK="1")
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--gpus", "2",
                          "--steps", "1", "--warmup", "3"], capture_output=True, text=True, timeout=300, cwd=ROOT,
                         env=env)
    assert out.returncode == 0 and out.stdout.strip() == ""


def _multi_worker(rank, ws, port, q):
    import torch.distributed as tdist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    tdist.init_process_group("gloo", rank=rank, world_size=ws)
    try:
        sys.path.insert(0, ROOT)
        import bench
        # per-rank device times (ms): the line must carry the max over ranks
        ring_ms = bench.reduce_max([1.0 + rank])[0]
        ctg_ms = bench.reduce_max([0.5 + rank])[0]
        payload = 128 << 20
        ring = {"ms": ring_ms, "chunk": 4 << 20, "depth": 0, "gbs_per_rank": payload / (ring_ms * 1e-3) / 1e9}
        sub = {"contiguous_same_bytes": {"ms": ctg_ms, "gbs_per_direction": payload / (ctg_ms * 1e-3) / 1e9},
               "nccl_mode_c3": {"error": "x"}, "c4_halo_ring": {"us_per_exchange": 50.0}}
        line = bench.assemble_multi_line(ws, 10, 3, payload, ring, sub, clocks={"sm_mhz": 1965},
                                         e2e={"value": 1.0, "unit": "GB/s", "h2d_bytes_per_step": 1,
                                              "d2h_bytes_per_step": 1}, replica={"gbs_per_rank": 5000.0})
        q.put((rank, json.dumps(line)))
    finally:
        tdist.destroy_process_group()


def test_multi_gpu_line_contract_gloo():
    """The N>1 line (world size 2 over gloo, fake device times): headline = whole-job
    bytes of the pairwise exchange per second from the max-over-ranks time, roofline
    against 900 GB/s per direction, the contiguous comparator beside it, side objects."""
    import multiprocessing as mp
    import socket
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_multi_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    out = dict(q.get(timeout=120) for _ in ps)
    for p in ps:
        p.join(60)
        assert p.exitcode == 0
    d = json.loads(out[0])
    assert out[0] == out[1]  # every rank computes the same line from the reduced times
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
              "vs_baseline", "dtype", "data", "config", "roofline", "gpu_launches", "transfer", "e2e", "clocks",
              "replica_pack_unpack"):
        assert k in d, k
    assert d["n_gpus"] == 2 and d["scaling"] == "weak" and d["ms_per_step"] == 2.0  # max over ranks
    per_dir = (128 << 20) / 2.0e-3 / 1e9
    assert abs(d["value"] - 2 * per_dir) < 0.2
    r = d["roofline"]
    assert r["bound"] == "nvlink" and r["peak"] == 900.0 and abs(r["frac"] - per_dir / 900.0) < 1e-3
    assert abs(d["config"]["of_contiguous"] - 0.75) < 1e-3  # ring 2.0 ms vs contiguous 1.5 ms
    assert "C3" in d["config"]["workload"]
    assert d["transfer"]["nccl_mode_c3"] == {"error": "x"}
