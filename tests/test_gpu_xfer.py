"""GPU transfer parity (T3/T4): dt_sendrecv must deliver exactly
oracle_unpack(rtype, oracle_pack(stype, sbuf)) into the receive layout and leave
every other byte untouched.  On one B200 the sender and
receiver are the same GPU: loopback inside one process (the paper's "1GPU"
case, [L26:c1686 §5.2.1]) and two processes on one GPU over CUDA IPC.  The
pipeline runs in fragments of `chunk` bytes through `depth` ring slots
([L18:c4394]-[L18:c5513 §4.1]); chunk sizes below the message size exercise
slot reuse and the ack flow control."""
import os
import socket

import numpy as np
import pytest

import oracle
from workloads import c1_submatrix, c2_lower_triangle, c3_block_cyclic, c5_particles, fill_bytes

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    os.environ.setdefault("DT_TIMEOUT_MS", "20000")
    return torch


def _loop_check(torch, comm, srec, sorg, sparent, rrec, rorg, rparent, scount=1, rcount=1, seed=3):
    from paper_conf_hpdc_wubvjd16_b200 import dt
    so, ro = oracle.from_recipe(srec), oracle.from_recipe(rrec)
    st, rt = dt.from_recipe(srec).commit(), dt.from_recipe(rrec).commit()
    sh = fill_bytes(sparent, seed)
    rh = np.full(rparent, 0xA5, dtype=np.uint8)
    exp = rh.copy()
    oracle.sendrecv(so, scount, sh, ro, rcount, exp, sorg, rorg)
    sd = torch.from_numpy(sh).cuda()
    rd = torch.from_numpy(rh).cuda()
    comm.sendrecv(sd, scount, st, comm.rank, rd, rcount, rt, comm.rank, sbuf_offset=sorg, rbuf_offset=rorg)
    torch.cuda.synchronize()
    comm.check()
    assert np.array_equal(rd.cpu().numpy(), exp)


@pytest.mark.parametrize("chunk,depth", [(64 << 10, 2), (256 << 10, 4), (1 << 20, 2), (4 << 20, 4)])
@pytest.mark.parametrize("ring", [True, False], ids=["ring", "fused"])
def test_loopback_block_cyclic(torch_cuda, chunk, depth, ring):
    from paper_conf_hpdc_wubvjd16_b200 import dt
    comm = dt.Comm(0, 1, 0, chunk_bytes=chunk, depth=depth, ring_loopback=ring)
    rec, org, parent = c3_block_cyclic(2048, 64)
    _loop_check(torch_cuda, comm, rec, org, parent, rec, org, parent)
    # repeated messages on the same channel reuse the ring (cumulative counters)
    for s in range(3):
        _loop_check(torch_cuda, comm, rec, org, parent, rec, org, parent, seed=10 + s)
    comm.free()


@pytest.mark.parametrize("wl", ["c3", "c4x"])
def test_loopback_system_scope(torch_cuda, wl, monkeypatch):
    """The peer-on-another-GPU configuration on one GPU (DT_XFER_SYS: system-scope flags,
    as across NVLink): the staged family's tiles leave with plain coalesced stores
    instead of TMA bulk stores into the peer's ring slot.  C3 (16-byte words) and the
    C4 x-face (4-byte words at a 2056-byte pitch), several fragments and one."""
    from paper_conf_hpdc_wubvjd16_b200 import dt
    from workloads import c4_face
    monkeypatch.setenv("DT_XFER_SYS", "1")
    for chunk in (256 << 10, 1 << 20):
        comm = dt.Comm(0, 1, 0, chunk_bytes=chunk, depth=0, ring_loopback=True)
        if wl == "c3":
            rec, org, parent = c3_block_cyclic(2048, 64)
            _loop_check(torch_cuda, comm, rec, org, parent, rec, org, parent)
        else:
            s, so, sp = c4_face("x-", 128)
            r, ro, rp = c4_face("x+", 128, ghost=True)
            _loop_check(torch_cuda, comm, s, so, sp, r, ro, rp)
        comm.free()


@pytest.mark.parametrize("ring", [True, False], ids=["ring", "fused"])
def test_loopback_different_types(torch_cuda, ring):
    """Same signature, different layouts (vector <-> contiguous, triangle -> packed;
    [L26:c4303 §5.2.2]); a receive larger than the message fills a prefix (A12).
    fused = f1, the datatype -> datatype copy without a ring."""
    from paper_conf_hpdc_wubvjd16_b200 import dt
    comm = dt.Comm(0, 1, 0, chunk_bytes=128 << 10, depth=3, ring_loopback=ring)
    v, vorg, vpar = c1_submatrix(256, 1024, 1, 1)
    contig = ("contiguous", 256 * 256, ("basic", "DOUBLE"))
    _loop_check(torch_cuda, comm, v, vorg, vpar, contig, 0, 256 * 256 * 8)
    _loop_check(torch_cuda, comm, contig, 0, 256 * 256 * 8, v, vorg, vpar)
    tri, _, tpar = c2_lower_triangle(600)
    n = 600 * 601 // 2
    _loop_check(torch_cuda, comm, tri, 0, tpar, ("contiguous", n + 100, ("basic", "DOUBLE")), 0, (n + 100) * 8)
    # message not a multiple of the receive layout's word size (ragged tail inside a staged fragment)
    _loop_check(torch_cuda, comm, ("contiguous", 125, ("basic", "DOUBLE")), 0, 1000,
                ("vector", 100, 2, 4, ("basic", "DOUBLE")), 0, 3200)
    # matrix transpose: column-major -> row-major as a vector of blocklength-1 columns ([L26:c4896 §5.2.3])
    m = 96
    rows = ("hvector", m, 1, 8, ("vector", m, 1, m, ("basic", "DOUBLE")))
    cols = ("contiguous", m * m, ("basic", "DOUBLE"))
    _loop_check(torch_cuda, comm, cols, 0, m * m * 8, rows, 0, m * m * 8)
    comm.free()


@pytest.mark.parametrize("ring", [True, False], ids=["ring", "fused"])
def test_loopback_short_blocks(torch_cuda, ring):
    from paper_conf_hpdc_wubvjd16_b200 import dt
    comm = dt.Comm(0, 1, 0, chunk_bytes=64 << 10, depth=2, ring_loopback=ring)
    rec, org, parent = c5_particles(1 << 20)
    _loop_check(torch_cuda, comm, rec, org, parent, rec, org, parent)
    comm.free()


def test_truncation_detected(torch_cuda):
    import torch

    from paper_conf_hpdc_wubvjd16_b200 import dt
    comm = dt.Comm(0, 1, 0, chunk_bytes=64 << 10, depth=2, ring_loopback=True)
    big = dt.Type.basic("DOUBLE").contiguous(1000).commit()
    small = dt.Type.basic("DOUBLE").contiguous(999).commit()
    s = torch.zeros(8000, dtype=torch.uint8, device="cuda")
    r = torch.full((8000,), 0xA5, dtype=torch.uint8, device="cuda")
    comm.sendrecv(s, 1, big, 0, r, 1, small, 0)
    torch.cuda.synchronize()
    with pytest.raises(dt.DTError) as e:
        comm.check()
    assert e.value.name == "DT_ERR_TRUNCATE"
    assert torch.all(r == 0xA5)
    # the channel stays usable afterwards
    s2 = torch.arange(8000, dtype=torch.int64, device="cuda").to(torch.uint8)
    comm.sendrecv(s2, 1, small, 0, r, 1, small, 0)
    torch.cuda.synchronize()
    comm.check()
    assert torch.equal(r[:7992], s2[:7992])
    # a message longer than the whole ring (16 x 64 KiB fragments through 2 slots): the
    # sender must be released by the receiver's abort instead of waiting for slots
    big = dt.Type.basic("BYTE").contiguous(1 << 20).commit()
    small = dt.Type.basic("BYTE").contiguous((1 << 20) - 1).commit()
    s3 = torch.randint(0, 255, (1 << 20,), dtype=torch.uint8, device="cuda")
    r3 = torch.full((1 << 20,), 0xA5, dtype=torch.uint8, device="cuda")
    comm.sendrecv(s3, 1, big, 0, r3, 1, small, 0)
    torch.cuda.synchronize()
    with pytest.raises(dt.DTError) as e:
        comm.check()
    assert e.value.name == "DT_ERR_TRUNCATE"
    assert torch.all(r3 == 0xA5)
    comm.sendrecv(s3, 1, big, 0, r3, 1, big, 0)
    torch.cuda.synchronize()
    comm.check()
    assert torch.equal(r3, s3)
    comm.free()


@pytest.mark.parametrize("ring", [True, False, "ce"], ids=["ring", "fused", "ce"])
def test_loopback_halo_all_faces(torch_cuda, ring):
    """1-rank periodic halo: the 12 transfers of one exchange in one group (through the
    ring kernel, the fused copy, or the copy-engine mode)."""
    import torch

    from paper_conf_hpdc_wubvjd16_b200 import dt
    from paper_conf_hpdc_wubvjd16_b200.halo import FACES, face_box, make_plan
    n, h = 64, 1
    L = n + 2 * h
    if ring == "ce":
        comm = dt.Comm(0, 1, 0, chunk_bytes=16 << 10, depth=2, mode=dt.XFER_CE)
    else:
        comm = dt.Comm(0, 1, 0, chunk_bytes=16 << 10, depth=2, ring_loopback=ring)
    plan = make_plan(0, n, h, dims=(1, 1, 1))
    A = np.full((L, L, L), 0xA5A5A5A5, dtype=np.uint32)
    z, y, x = np.meshgrid(np.arange(n), np.arange(n), np.arange(n), indexing="ij")
    A[h:h + n, h:h + n, h:h + n] = (z * 1000000 + y * 1000 + x).astype(np.uint32)
    buf = torch.from_numpy(A.view(np.uint8).reshape(-1).copy()).cuda()
    plan.exchange(comm, buf)
    torch.cuda.synchronize()
    comm.check()
    B = buf.cpu().numpy().view(np.uint32).reshape(L, L, L)
    for f in FACES:
        sub, st = face_box(f, n, h, ghost=True)
        zz, yy, xx = np.meshgrid(*[np.arange(s, s + k) for s, k in zip(st, sub)], indexing="ij")
        exp = (((zz - h) % n) * 1000000 + ((yy - h) % n) * 1000 + ((xx - h) % n)).astype(np.uint32)
        assert np.array_equal(B[zz, yy, xx], exp), f
    comm.free()


def test_nccl_mode_loopback(torch_cuda):
    from paper_conf_hpdc_wubvjd16_b200 import dt
    try:
        nid = dt.Comm.nccl_unique_id()
    except dt.DTError as e:
        pytest.skip(f"NCCL unavailable: {e}")
    comm = dt.Comm(0, 1, 0, chunk_bytes=256 << 10, depth=2, mode=dt.XFER_NCCL, nccl_id=nid)
    rec, org, parent = c3_block_cyclic(1024, 64)
    _loop_check(torch_cuda, comm, rec, org, parent, rec, org, parent)
    comm.free()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _ipc_worker(rank, port, q, mode=0):
    try:
        import torch
        import torch.distributed as tdist
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        os.environ.setdefault("DT_TIMEOUT_MS", "60000")
        tdist.init_process_group("gloo", rank=rank, world_size=2)
        torch.cuda.set_device(0)
        from paper_conf_hpdc_wubvjd16_b200 import dt
        comm = dt.Comm.from_process_group(device=0, chunk_bytes=256 << 10, depth=2, ctas=4, mode=mode)
        rec, org, parent = c2_lower_triangle(1024)
        t = dt.from_recipe(rec).commit()
        mine = fill_bytes(parent, 100 + rank)
        other = fill_bytes(parent, 100 + (1 - rank))
        sd = torch.from_numpy(mine).cuda()
        rd = torch.full((parent,), 0xA5, dtype=torch.uint8, device="cuda")
        comm.sendrecv(sd, 1, t, 1 - rank, rd, 1, t, 1 - rank)
        torch.cuda.synchronize()
        comm.check()
        exp = np.full(parent, 0xA5, dtype=np.uint8)
        ot = oracle.from_recipe(rec)
        oracle.sendrecv(ot, 1, other, ot, 1, exp)
        ok = bool(np.array_equal(rd.cpu().numpy(), exp))
        tdist.barrier()
        comm.free()
        q.put((rank, ok))
        tdist.destroy_process_group()
    except Exception as e:  # noqa: BLE001
        import traceback
        q.put((rank, traceback.format_exc() + repr(e)))


@pytest.mark.parametrize("mode", [0, 2], ids=["p2p", "ce"])
def test_two_processes_one_gpu_ipc(torch_cuda, mode):
    """Two ranks (processes) exchange triangles through IPC-mapped rings on one GPU (the
    P2P kernel, or the copy-engine mode: staging, cudaMemcpyAsync into the peer ring,
    stream-ordered flag kernels)."""
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_ipc_worker, args=(r, port, q, mode)) for r in range(2)]
    for p in ps:
        p.start()
    res = [q.get(timeout=300) for _ in ps]
    for p in ps:
        p.join(timeout=60)
    for rank, ok in res:
        assert ok is True, (rank, ok)


def test_fused_copy_direct(torch_cuda):
    """dt_copy (f1) directly: transpose via blocklength-1 vectors ([L26:c4896 §5.2.3]),
    vector <-> contiguous ([L26:c4303 §5.2.2]), triangle -> block-cyclic-shaped
    layouts of equal size, both kernel families (forced), truncation, overlap."""
    import torch

    from paper_conf_hpdc_wubvjd16_b200 import dt
    m = 200
    cases = [
        (("contiguous", m * m, ("basic", "DOUBLE")), 0, m * m * 8,
         ("hvector", m, 1, 8, ("vector", m, 1, m, ("basic", "DOUBLE"))), 0, m * m * 8),
        (c1_submatrix(128, 512, 3, 5)[:3] + (("contiguous", 128 * 128, ("basic", "DOUBLE")), 0, 128 * 128 * 8)),
        (c2_lower_triangle(257)[:3] + c5_particles(257 * 258 // 2 * 8)[:3]),
        (c5_particles(56 * 3000)[:3] + (("contiguous", 3000 * 14, ("basic", "INT32")), 0, 3000 * 56)),
    ]
    for force in ("", "1", "2"):
        os.environ["DT_FORCE_KERNEL"] = force
        for i, (srec, sorg, spar, rrec, rorg, rpar) in enumerate(cases):
            so, ro = oracle.from_recipe(srec), oracle.from_recipe(rrec)
            if so.size > ro.size:
                continue
            st, rt = dt.from_recipe(srec).commit(), dt.from_recipe(rrec).commit()
            sh = fill_bytes(spar, 70 + i)
            exp = np.full(rpar, 0xA5, dtype=np.uint8)
            oracle.sendrecv(so, 1, sh, ro, 1, exp, sorg, rorg)
            rd = torch.full((rpar,), 0xA5, dtype=torch.uint8, device="cuda")
            dt.copy(st, 1, torch.from_numpy(sh).cuda(), rt, 1, rd, src_offset=sorg, dst_offset=rorg)
            torch.cuda.synchronize()
            assert np.array_equal(rd.cpu().numpy(), exp), (force, i)
    os.environ.pop("DT_FORCE_KERNEL", None)
    a = dt.Type.basic("DOUBLE").contiguous(10).commit()
    b = dt.Type.basic("DOUBLE").contiguous(9).commit()
    x = torch.zeros(80, dtype=torch.uint8, device="cuda")
    with pytest.raises(dt.DTError) as e:
        dt.copy(a, 1, x, b, 1, x)
    assert e.value.name == "DT_ERR_TRUNCATE"
    ov = dt.Type.basic("INT32").vector(4, 3, 2).commit()
    with pytest.raises(dt.DTError) as e:
        dt.copy(dt.Type.basic("INT32").contiguous(12).commit(), 1, x, ov, 1, x)
    assert e.value.name == "DT_ERR_OVERLAP"


# ------------------------------------------------------------------ persistent direct plans (dt_xplan, f1 across GPUs)
def _direct_case(torch, srec, sorg, spar, rrec, rorg, rpar, seed):
    """(send tensor, receive tensor, expected receive bytes) for one send -> receive."""
    so, ro = oracle.from_recipe(srec), oracle.from_recipe(rrec)
    sh = fill_bytes(spar, seed)
    exp = np.full(rpar, 0xA5, dtype=np.uint8)
    oracle.sendrecv(so, 1, sh, ro, 1, exp, sorg, rorg)
    return torch.from_numpy(sh).cuda(), torch.full((rpar,), 0xA5, dtype=torch.uint8, device="cuda"), exp


def test_direct_plan_single_rank(torch_cuda):
    """A 1-rank plan of several sends-to-self with different send/receive types and
    every copy family (long runs, word tables, staged): repeated starts reuse the
    flags (sequence numbers), each start moves the CURRENT source bytes."""
    import torch

    from paper_conf_hpdc_wubvjd16_b200 import dt
    comm = dt.Comm(0, 1, 0)
    pairs = [c3_block_cyclic(1024, 64)[:3] * 2,
             c2_lower_triangle(257)[:3] + c5_particles(257 * 258 // 2 * 8)[:3],
             c5_particles(56 * 3000)[:3] + (("contiguous", 3000 * 14, ("basic", "INT32")), 0, 3000 * 56),
             c1_submatrix(128, 512, 3, 5)[:3] + (("contiguous", 128 * 128, ("basic", "DOUBLE")), 0, 128 * 128 * 8)]
    for rnd in range(3):
        sends, recvs, exps, bufs = [], [], [], []
        for i, (sr, so_, sp, rr, ro_, rp) in enumerate(pairs):
            sd, rd, exp = _direct_case(torch, sr, so_, sp, rr, ro_, rp, 40 + i + 10 * rnd)
            st, rt = dt.from_recipe(sr).commit(), dt.from_recipe(rr).commit()
            sends.append((sd.data_ptr() + so_, 1, st, 0, i))
            recvs.append((rd.data_ptr() + ro_, 1, rt, 0, i))
            exps.append(exp)
            bufs.append((sd, rd, st, rt))
        plan = dt.XPlan.local(comm, sends, recvs)
        for _ in range(2):  # the second start re-sends the same bytes into the same layouts
            plan.start()
            torch.cuda.synchronize()
            plan.check()
        for (sd, rd, _, _), exp in zip(bufs, exps):
            assert np.array_equal(rd.cpu().numpy(), exp), rnd
        plan.free()
    comm.free()


def test_direct_plan_halo_single_rank(torch_cuda):
    """1-rank periodic halo as one direct plan (12 ops, one kernel per exchange)."""
    import torch

    from paper_conf_hpdc_wubvjd16_b200 import dt
    from paper_conf_hpdc_wubvjd16_b200.halo import FACES, face_box, make_plan
    n, h = 64, 1
    L = n + 2 * h
    comm = dt.Comm(0, 1, 0)
    hp = make_plan(0, n, h, dims=(1, 1, 1))
    A = np.full((L, L, L), 0xA5A5A5A5, dtype=np.uint32)
    z, y, x = np.meshgrid(np.arange(n), np.arange(n), np.arange(n), indexing="ij")
    A[h:h + n, h:h + n, h:h + n] = (z * 1000000 + y * 1000 + x).astype(np.uint32)
    buf = torch.from_numpy(A.view(np.uint8).reshape(-1).copy()).cuda()
    xp = hp.direct_plan(comm, buf, single_rank=True)
    for _ in range(3):
        xp.start()
    torch.cuda.synchronize()
    xp.check()
    B = buf.cpu().numpy().view(np.uint32).reshape(L, L, L)
    for f in FACES:
        sub, st = face_box(f, n, h, ghost=True)
        zz, yy, xx = np.meshgrid(*[np.arange(s, s + k) for s, k in zip(st, sub)], indexing="ij")
        exp = (((zz - h) % n) * 1000000 + ((yy - h) % n) * 1000 + ((xx - h) % n)).astype(np.uint32)
        assert np.array_equal(B[zz, yy, xx], exp), f
    # the interior is untouched
    assert np.array_equal(B[h:h + n, h:h + n, h:h + n], A[h:h + n, h:h + n, h:h + n])
    xp.free()
    comm.free()


@pytest.mark.parametrize("ring", [True, False], ids=["ring", "fused"])
def test_hybrid_halo_single_rank(torch_cuda, ring):
    """1-rank periodic halo, hybrid: y/z faces through a direct plan on the main
    stream, x faces through the ring group on a side stream joined by an event."""
    import torch

    from paper_conf_hpdc_wubvjd16_b200 import dt
    from paper_conf_hpdc_wubvjd16_b200.halo import FACES, face_box, make_plan
    n, h = 48, 1
    L = n + 2 * h
    comm = dt.Comm(0, 1, 0, chunk_bytes=8 << 10, depth=2, ring_loopback=ring)
    hp = make_plan(0, n, h, dims=(1, 1, 1))
    assert [f for _, f, _ in hp.ops(("x-", "x+"))] == ["x-", "x+", "x+", "x-"]
    A = np.full((L, L, L), 0xA5A5A5A5, dtype=np.uint32)
    z, y, x = np.meshgrid(np.arange(n), np.arange(n), np.arange(n), indexing="ij")
    A[h:h + n, h:h + n, h:h + n] = (z * 1000000 + y * 1000 + x).astype(np.uint32)
    buf = torch.from_numpy(A.view(np.uint8).reshape(-1).copy()).cuda()
    s = torch.cuda.current_stream()
    run = hp.hybrid(comm, buf, s, single_rank=True)
    for _ in range(3):
        run()
    torch.cuda.synchronize()
    run.check()
    B = buf.cpu().numpy().view(np.uint32).reshape(L, L, L)
    for f in FACES:
        sub, st = face_box(f, n, h, ghost=True)
        zz, yy, xx = np.meshgrid(*[np.arange(s_, s_ + k) for s_, k in zip(st, sub)], indexing="ij")
        exp = (((zz - h) % n) * 1000000 + ((yy - h) % n) * 1000 + ((xx - h) % n)).astype(np.uint32)
        assert np.array_equal(B[zz, yy, xx], exp), f
    assert np.array_equal(B[h:h + n, h:h + n, h:h + n], A[h:h + n, h:h + n, h:h + n])
    # edges and corners (outside every face box) are untouched
    assert np.all(B[0, 0, :] == 0xA5A5A5A5) and np.all(B[:, 0, 0] == 0xA5A5A5A5)
    run.plan.free()
    comm.free()


@pytest.mark.parametrize("ring", [True, False], ids=["ring", "fused"])
def test_halo_exchange_face_subset(torch_cuda, ring):
    """exchange(faces=xs) posts only the x transfers: the x ghost layers are filled,
    the y/z ghost layers keep their poison (the subset was ignored)."""
    import torch

    from paper_conf_hpdc_wubvjd16_b200 import dt
    from paper_conf_hpdc_wubvjd16_b200.halo import FACES, face_box, make_plan
    n, h = 40, 1
    L = n + 2 * h
    comm = dt.Comm(0, 1, 0, chunk_bytes=8 << 10, depth=2, ring_loopback=ring)
    hp = make_plan(0, n, h, dims=(1, 1, 1))
    A = np.full((L, L, L), 0xA5A5A5A5, dtype=np.uint32)
    z, y, x = np.meshgrid(np.arange(n), np.arange(n), np.arange(n), indexing="ij")
    A[h:h + n, h:h + n, h:h + n] = (z * 1000000 + y * 1000 + x).astype(np.uint32)
    buf = torch.from_numpy(A.view(np.uint8).reshape(-1).copy()).cuda()
    hp.exchange(comm, buf, faces=("x-", "x+"))
    torch.cuda.synchronize()
    comm.check()
    B = buf.cpu().numpy().view(np.uint32).reshape(L, L, L)
    for f in FACES:
        sub, st = face_box(f, n, h, ghost=True)
        zz, yy, xx = np.meshgrid(*[np.arange(s_, s_ + k) for s_, k in zip(st, sub)], indexing="ij")
        if f[0] == "x":
            exp = (((zz - h) % n) * 1000000 + ((yy - h) % n) * 1000 + ((xx - h) % n)).astype(np.uint32)
            assert np.array_equal(B[zz, yy, xx], exp), f
        else:
            assert np.all(B[zz, yy, xx] == 0xA5A5A5A5), f
    comm.free()


def test_direct_plan_errors(torch_cuda):
    import torch

    from paper_conf_hpdc_wubvjd16_b200 import dt
    comm = dt.Comm(0, 1, 0)
    x = torch.zeros(4096, dtype=torch.uint8, device="cuda")
    a = dt.Type.basic("DOUBLE").contiguous(10).commit()
    b = dt.Type.basic("DOUBLE").contiguous(9).commit()
    with pytest.raises(dt.DTError) as e:   # 80 bytes into a 72-byte receive: at connect, before any byte moves
        dt.XPlan.local(comm, [(x, 1, a, 0, 7)], [(x.data_ptr() + 1024, 1, b, 0, 7)])
    assert e.value.name == "DT_ERR_TRUNCATE"
    ov = dt.Type.basic("INT32").vector(4, 3, 2).commit()
    with pytest.raises(dt.DTError) as e:
        dt.XPlan.local(comm, [], [(x, 1, ov, 0, 1)])
    assert e.value.name == "DT_ERR_OVERLAP"
    with pytest.raises(dt.DTError) as e:   # no receive with this tag
        dt.XPlan.local(comm, [(x, 1, a, 0, 1)], [(x.data_ptr() + 1024, 1, a, 0, 2)])
    assert e.value.name == "DT_ERR_ARG"
    comm.free()


def _direct_worker(rank, port, q):
    try:
        import torch
        import torch.distributed as tdist
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        os.environ.setdefault("DT_TIMEOUT_MS", "60000")
        tdist.init_process_group("gloo", rank=rank, world_size=2)
        torch.cuda.set_device(0)
        from paper_conf_hpdc_wubvjd16_b200 import dt
        comm = dt.Comm.from_process_group(device=0)
        # rank 0 sends its lower triangle into rank 1's block-cyclic-shaped receive, rank 1
        # sends its block-cyclic submatrix into rank 0's contiguous receive (types differ)
        tri, torg, tpar = c2_lower_triangle(512)
        bc, borg, bpar = c3_block_cyclic(1024, 64)
        ot, ob = oracle.from_recipe(tri), oracle.from_recipe(bc)
        ctg = ("contiguous", ob.size, ("basic", "BYTE"))
        oc = oracle.from_recipe(ctg)
        T, B, Cg = (dt.from_recipe(r).commit() for r in (tri, bc, ctg))
        mine = torch.from_numpy(fill_bytes(max(tpar, bpar), 300 + rank)).cuda()
        rbuf = torch.full((max(bpar, ob.size) + 64,), 0xA5, dtype=torch.uint8, device="cuda")
        if rank == 0:
            sends = [(mine.data_ptr() + torg, 1, T, 1, 5)]
            recvs = [(rbuf, 1, Cg, 1, 9)]
        else:
            sends = [(mine.data_ptr() + borg, 1, B, 0, 9)]
            # receive the 512^2 triangle's bytes into the first bytes of a block-cyclic layout
            recvs = [(rbuf.data_ptr() + borg, 1, B, 0, 5)]
        plan = dt.XPlan.from_process_group(comm, sends, recvs)
        for _ in range(2):
            plan.start()
        torch.cuda.synchronize()
        plan.check()
        other = fill_bytes(max(tpar, bpar), 300 + (1 - rank))
        exp = np.full(rbuf.numel(), 0xA5, dtype=np.uint8)
        if rank == 0:
            oracle.sendrecv(ob, 1, other, oc, 1, exp, borg, 0)
        else:
            oracle.sendrecv(ot, 1, other, ob, 1, exp, torg, borg)
        ok = bool(np.array_equal(rbuf.cpu().numpy(), exp))
        tdist.barrier()
        plan.free()
        comm.free()
        q.put((rank, ok))
        tdist.destroy_process_group()
    except Exception as e:  # noqa: BLE001
        import traceback
        q.put((rank, traceback.format_exc() + repr(e)))


def test_direct_plan_two_processes_ipc(torch_cuda):
    """Two ranks (processes) with different send/receive types: each rank's kernel
    writes straight into the other process's buffer through CUDA IPC."""
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_direct_worker, args=(r, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = [q.get(timeout=300) for _ in ps]
    for p in ps:
        p.join(timeout=60)
    for rank, ok in res:
        assert ok is True, (rank, ok)


@pytest.mark.parametrize("chunk", [16 << 10, 256 << 10])
def test_ring_record_spans(torch_cuda, chunk):
    """Record-span fragments inside the ring pipeline (sender packs whole-record 16-byte
    loads into the ring slot, receiver scatters covered chunks): particles and
    other dense-record layouts against a contiguous peer, both directions, count 2."""
    from paper_conf_hpdc_wubvjd16_b200 import dt
    from tests.test_gpu_parity import REC_TYPES
    comm = dt.Comm(0, 1, 0, chunk_bytes=chunk, depth=2, ring_loopback=True)
    for name in sorted(REC_TYPES):
        rec, org, parent = REC_TYPES[name]()
        size = oracle.from_recipe(rec).size
        ctg = ("contiguous", 2 * size, ("basic", "BYTE"))
        ext = oracle.from_recipe(rec).extent
        _loop_check(torch_cuda, comm, rec, org, parent + ext, ctg, 0, 2 * size, scount=2, rcount=1)
        _loop_check(torch_cuda, comm, ctg, 0, 2 * size, rec, org, parent + ext, scount=1, rcount=2)
        _loop_check(torch_cuda, comm, rec, org, parent, rec, org, parent)
    comm.free()


@pytest.mark.parametrize("chunk", [16 << 10, 1 << 20])
def test_ring_block_spans(torch_cuda, chunk):
    """Block-span fragments inside the ring pipeline (C5b-like irregular lists of short
    blocks: 32-block windows per warp, span loads, packed/span word maps) against a
    contiguous peer in both directions and type to itself, count 2 (element wrap)."""
    from paper_conf_hpdc_wubvjd16_b200 import dt
    from tests.test_gpu_parity import SPAN_TYPES
    from workloads import c5b_irregular
    comm = dt.Comm(0, 1, 0, chunk_bytes=chunk, depth=2, ring_loopback=True)
    cases = dict(SPAN_TYPES)
    cases["c5b"] = c5b_irregular(3 << 20)
    for name in sorted(cases):
        rec, org, parent = cases[name]
        size = oracle.from_recipe(rec).size
        ext = oracle.from_recipe(rec).extent
        ctg = ("contiguous", 2 * size, ("basic", "BYTE"))
        _loop_check(torch_cuda, comm, rec, org, parent + ext, ctg, 0, 2 * size, scount=2, rcount=1)
        _loop_check(torch_cuda, comm, ctg, 0, 2 * size, rec, org, parent + ext, scount=1, rcount=2)
        _loop_check(torch_cuda, comm, rec, org, parent, rec, org, parent)
    comm.free()


@pytest.mark.parametrize("rep,depth", [("1", 4), ("2", 4), ("2", 8), ("4", 8), ("2", 2)])
def test_ring_replicas(torch_cuda, rep, depth, monkeypatch):
    """Replicated sub-rings (rep CTAs per sub-ring taking alternate fragments, announced in
    the header; the receiver maps its CTAs onto the replicas): bit-exact for every
    replica/depth combination, including the fallback to one replica when a replica
    would own a single slot, with repeated messages on the same channel."""
    from paper_conf_hpdc_wubvjd16_b200 import dt
    monkeypatch.setenv("DT_XFER_REP", rep)
    comm = dt.Comm(0, 1, 0, chunk_bytes=256 << 10, depth=depth, ring_loopback=True)
    rec, org, parent = c3_block_cyclic(2048, 64)
    for s in range(2):
        _loop_check(torch_cuda, comm, rec, org, parent, rec, org, parent, seed=20 + s)
    rec5, org5, parent5 = c5_particles(3 << 20)
    _loop_check(torch_cuda, comm, rec5, org5, parent5, rec5, org5, parent5, seed=7)
    comm.free()


@pytest.mark.parametrize("chunk", [1 << 20, 4 << 20])
def test_full_size_c3_exchange_sampled(torch_cuda, chunk):
    """BASELINE configs C3 at full size in the launch configuration the bench times
    (8192^2 f64, nb 64, 128 MiB per direction, auto depth, 1 and 4 MiB fragments):
    sampled received bytes against the oracle's per-position addresses, gap bytes of the
    receive layout untouched, repeated exchanges on the same channel."""
    import torch

    from paper_conf_hpdc_wubvjd16_b200 import dt
    rec, org, parent = c3_block_cyclic(8192, 64)
    ot = oracle.from_recipe(rec)
    t = dt.from_recipe(rec).commit()
    comm = dt.Comm(0, 1, 0, chunk_bytes=chunk, depth=0, ring_loopback=True)
    src_h = fill_bytes(parent, 0x5EED0003)
    A = torch.from_numpy(src_h).cuda()
    B = torch.full((parent,), 0xA5, dtype=torch.uint8, device="cuda")
    for _ in range(3):
        comm.sendrecv(A, 1, t, 0, B, 1, t, 0, sbuf_offset=org, rbuf_offset=org)
    torch.cuda.synchronize()
    comm.check()
    rng = np.random.default_rng(3)
    n = ot.size
    ps = np.unique(np.concatenate([rng.integers(0, n, size=300000), [0, n - 1]]))
    addr = org + oracle.addr_of(ot, 1, ps)
    got = B[torch.from_numpy(addr).cuda()].cpu().numpy()
    assert np.array_equal(got, src_h[addr])
    # bytes outside the typemap: the other processes' blocks of the block-cyclic layout
    # (rows nb..2nb of each owned column) keep their poison
    gaps = org + np.arange(64) * 8 + 64 * 8
    assert np.all(B[torch.from_numpy(gaps).cuda()].cpu().numpy() == 0xA5)
    comm.free()


def test_full_size_c4_halo_ring(torch_cuda):
    """C4 at full size (512^3 f32 per rank, ghost width 1, periodic on one GPU), all 12
    transfers through the ring group as the bench times them: every ghost cell equals
    the periodic neighbour's interior value (closed form), the interior is untouched."""
    import torch

    from paper_conf_hpdc_wubvjd16_b200 import dt
    from paper_conf_hpdc_wubvjd16_b200.halo import make_plan
    n, h = 512, 1
    L = n + 2 * h
    comm = dt.Comm(0, 1, 0, chunk_bytes=1 << 20, depth=0, ring_loopback=True)
    plan = make_plan(0, n, h, dims=(1, 1, 1))
    buf = torch.empty(L ** 3 * 4, dtype=torch.uint8, device="cuda")
    A = buf.view(torch.int32).view(L, L, L)
    A.random_(0, 1 << 30)
    before = A[h:h + n, h:h + n, h:h + n].clone()
    for _ in range(2):
        plan.exchange(comm, buf)
    torch.cuda.synchronize()
    comm.check()
    assert torch.equal(A[h:h + n, h:h + n, 0], A[h:h + n, h:h + n, n])          # x- ghost = x+ boundary
    assert torch.equal(A[h:h + n, h:h + n, L - 1], A[h:h + n, h:h + n, h])      # x+ ghost = x- boundary
    assert torch.equal(A[h:h + n, 0, h:h + n], A[h:h + n, n, h:h + n])
    assert torch.equal(A[h:h + n, L - 1, h:h + n], A[h:h + n, h, h:h + n])
    assert torch.equal(A[0, h:h + n, h:h + n], A[n, h:h + n, h:h + n])
    assert torch.equal(A[L - 1, h:h + n, h:h + n], A[h, h:h + n, h:h + n])
    assert torch.equal(A[h:h + n, h:h + n, h:h + n], before)
    comm.free()


def test_ring_exchange_graph_replay(torch_cuda):
    """Sequence numbers live on the device, so ring exchanges captured once in a CUDA
    graph replay correctly: every replay moves the current source bytes (the paper's
    persistent exchange of a halo/stencil loop without per-message host work)."""
    import torch

    from paper_conf_hpdc_wubvjd16_b200 import dt
    rec, org, parent = c3_block_cyclic(2048, 64)
    ot = oracle.from_recipe(rec)
    t = dt.from_recipe(rec).commit()
    v = dt.Type.basic("INT32").contiguous(1000).commit()
    comm = dt.Comm(0, 1, 0, chunk_bytes=256 << 10, depth=0, ring_loopback=True)
    A = torch.zeros(parent, dtype=torch.uint8, device="cuda")
    B = torch.full((parent,), 0xA5, dtype=torch.uint8, device="cuda")
    a2 = torch.zeros(4000, dtype=torch.uint8, device="cuda")
    b2 = torch.zeros(4000, dtype=torch.uint8, device="cuda")
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        for _ in range(2):  # warm up: descriptors, word tables, attributes
            comm.sendrecv(A, 1, t, 0, B, 1, t, 0, sbuf_offset=org, rbuf_offset=org, stream=s)
            comm.sendrecv(a2, 1, v, 0, b2, 1, v, 0, stream=s)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        comm.sendrecv(A, 1, t, 0, B, 1, t, 0, sbuf_offset=org, rbuf_offset=org, stream=s)
        comm.sendrecv(a2, 1, v, 0, b2, 1, v, 0, stream=s)
    for r in range(4):
        src_h = fill_bytes(parent, 100 + r)
        A.copy_(torch.from_numpy(src_h))
        a2.copy_(torch.from_numpy(fill_bytes(4000, 200 + r)))
        g.replay()
        torch.cuda.synchronize()
        comm.check()
        exp_b = B.cpu().numpy().copy()
        oracle.sendrecv(ot, 1, src_h, ot, 1, exp_b, org, org)
        assert np.array_equal(B.cpu().numpy(), exp_b), r
        assert torch.equal(b2, a2), r
    comm.free()


@pytest.mark.parametrize("chunk,depth", [(64 << 10, 2), (256 << 10, 4), (1 << 20, 0)])
def test_copy_engine_mode_loopback(torch_cuda, chunk, depth):
    """DT_XFER_CE ([L20:c4255 §4.1] receiver staging with the copy engine as the wire):
    block-cyclic exchanges repeated on one channel (ring slots reused across rounds and
    messages), different send/receive layouts, short-block particles, and truncation
    (reported by dt_sendrecv; the channel stays usable)."""
    from paper_conf_hpdc_wubvjd16_b200 import dt
    comm = dt.Comm(0, 1, 0, chunk_bytes=chunk, depth=depth, mode=dt.XFER_CE)
    rec, org, parent = c3_block_cyclic(2048, 64)
    for s_ in range(3):
        _loop_check(torch_cuda, comm, rec, org, parent, rec, org, parent, seed=20 + s_)
    v, vorg, vpar = c1_submatrix(256, 1024, 1, 1)
    contig = ("contiguous", 256 * 256, ("basic", "DOUBLE"))
    _loop_check(torch_cuda, comm, v, vorg, vpar, contig, 0, 256 * 256 * 8)
    tri, _, tpar = c2_lower_triangle(600)
    n = 600 * 601 // 2
    _loop_check(torch_cuda, comm, tri, 0, tpar, ("contiguous", n + 100, ("basic", "DOUBLE")), 0, (n + 100) * 8)
    prec, porg, ppar = c5_particles(1 << 20)
    _loop_check(torch_cuda, comm, prec, porg, ppar, prec, porg, ppar)
    import torch
    big = dt.Type.basic("BYTE").contiguous(3 * chunk + 5).commit()
    small = dt.Type.basic("BYTE").contiguous(3 * chunk).commit()
    sb = torch.randint(0, 255, (3 * chunk + 5,), dtype=torch.uint8, device="cuda")
    rb = torch.full((3 * chunk + 5,), 0xA5, dtype=torch.uint8, device="cuda")
    with pytest.raises(dt.DTError) as e:
        comm.sendrecv(sb, 1, big, 0, rb, 1, small, 0)
    assert e.value.name == "DT_ERR_TRUNCATE"
    torch.cuda.synchronize()
    assert torch.all(rb == 0xA5)
    _loop_check(torch_cuda, comm, rec, org, parent, rec, org, parent, seed=30)
    comm.free()
