"""N>1 host logic on CPU (world_size 2, gloo): the handle/unique-id exchange
the transfer engine bootstraps with, and the 3D halo exchange plan (config C4,
SHOC-style boundaries [L14:c1929 §3], reading A17) run end to end with the
oracle doing the pack/unpack and gloo carrying the packed bytes.  Messages
between one pair are matched first-posted-first-matched, the same rule libdt's
channels implement, so a correct ghost layer here validates the posting order
that the GPU path uses."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _init(rank, ws, port):
    import torch.distributed as tdist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    tdist.init_process_group("gloo", rank=rank, world_size=ws)
    return tdist


def _value(gz, gy, gx):
    """closed-form cell content: hash of global coordinates (uint32)."""
    v = (np.uint64(gz) * np.uint64(73856093)) ^ (np.uint64(gy) * np.uint64(19349663)) ^ (np.uint64(gx) * np.uint64(83492791))
    return (v & np.uint64(0xFFFFFFFF)).astype(np.uint32)


def _worker_blobs(rank, ws, port, q):
    try:
        tdist = _init(rank, ws, port)
        from paper_conf_hpdc_wubvjd16_b200.dt import broadcast_id, exchange_blobs
        blob = bytes([rank]) * 40
        allb = exchange_blobs(blob)
        nid = broadcast_id(b"\x07" * 128 if rank == 0 else None)
        q.put((rank, allb, nid))
        tdist.destroy_process_group()
    except Exception as e:  # noqa: BLE001
        q.put((rank, repr(e), None))


def test_handle_exchange_two_ranks():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker_blobs, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = [q.get(timeout=120) for _ in ps]
    for p in ps:
        p.join(timeout=60)
    for rank, allb, nid in res:
        assert allb == bytes([0]) * 40 + bytes([1]) * 40, (rank, allb)
        assert nid == b"\x07" * 128


def _worker_halo(rank, ws, port, dims, n, q):
    try:
        tdist = _init(rank, ws, port)
        import torch

        import oracle
        from paper_conf_hpdc_wubvjd16_b200.halo import OPPOSITE, HaloPlan, grid_coords, neighbour
        from workloads import c4_face
        h = 1
        L = n + 2 * h
        pz, py, px = grid_coords(rank, dims)
        A = np.full((L, L, L), 0xA5A5A5A5, dtype=np.uint32)
        z, y, x = np.meshgrid(np.arange(n), np.arange(n), np.arange(n), indexing="ij")
        A[h:h + n, h:h + n, h:h + n] = _value(pz * n + z, py * n + y, px * n + x)
        buf = A.view(np.uint8).reshape(-1)
        plan = HaloPlan(n, h, dims, rank, {}, {})
        sent, recvd = {}, {}
        reqs, local = [], {}
        incoming = []
        for kind, face, peer in plan.ops():
            if kind == "send":
                ot = oracle.from_recipe(c4_face(face, n, h, ghost=False)[0])
                data = oracle.pack(ot, 1, buf)
                k = sent.get(peer, 0)
                sent[peer] = k + 1
                if peer == rank:
                    local.setdefault(k, data)
                else:
                    reqs.append(tdist.isend(torch.from_numpy(data.copy()), dst=peer, tag=k))
            else:
                k = recvd.get(peer, 0)
                recvd[peer] = k + 1
                incoming.append((face, peer, k))
        for face, peer, k in incoming:
            ot = oracle.from_recipe(c4_face(face, n, h, ghost=True)[0])
            if peer == rank:
                data = local[k]
            else:
                t = torch.empty(ot.size, dtype=torch.uint8)
                tdist.recv(t, src=peer, tag=k)
                data = t.numpy()
            oracle.unpack(ot, 1, data, buf)
        for r in reqs:
            r.wait()
        # every ghost cell equals the closed form at the periodically wrapped global coords
        N = [d * n for d in dims]
        bad = 0
        for face in ("x-", "x+", "y-", "y+", "z-", "z+"):
            sub, st = plan_box(face, n, h)
            zz, yy, xx = np.meshgrid(*[np.arange(s, s + k) for s, k in zip(st, sub)], indexing="ij")
            g = [(pz * n + zz - h) % N[0], (py * n + yy - h) % N[1], (px * n + xx - h) % N[2]]
            bad += int(np.sum(A[zz, yy, xx] != _value(*g)))
        del OPPOSITE, neighbour
        q.put((rank, bad))
        tdist.destroy_process_group()
    except Exception as e:  # noqa: BLE001
        import traceback
        q.put((rank, traceback.format_exc() + repr(e)))


def plan_box(face, n, h):
    from paper_conf_hpdc_wubvjd16_b200.halo import face_box
    return face_box(face, n, h, ghost=True)


@pytest.mark.parametrize("dims", [(1, 1, 2), (1, 2, 1), (2, 1, 1)])
def test_halo_plan_two_ranks(dims):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker_halo, args=(r, 2, port, dims, 6, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = [q.get(timeout=180) for _ in ps]
    for p in ps:
        p.join(timeout=60)
    for rank, bad in res:
        assert bad == 0, (rank, bad)


def test_halo_plan_geometry():
    from paper_conf_hpdc_wubvjd16_b200.halo import FACES, OPPOSITE, grid_coords, grid_rank, neighbour
    dims = (2, 2, 2)
    for r in range(8):
        assert grid_rank(grid_coords(r, dims), dims) == r
        for f in FACES:
            assert neighbour(neighbour(r, f, dims), OPPOSITE[f], dims) == r
    # 2x2x2 periodic: both x neighbours are the same rank (3 distinct peers, reading A17)
    assert len({neighbour(0, f, dims) for f in FACES}) == 3


def test_halo_ops_face_subsets():
    """The hybrid exchange splits one exchange into face subsets closed under
    OPPOSITE; the subsets' ops partition the full exchange's ops, and each subset
    keeps the global posting order (sender's face in FACES order)."""
    from paper_conf_hpdc_wubvjd16_b200.halo import FACES, OPPOSITE, HaloPlan
    for dims in [(2, 2, 2), (1, 2, 2), (1, 1, 2)]:
        for r in range(dims[0] * dims[1] * dims[2]):
            hp = HaloPlan(8, 1, dims, r, {}, {})
            full = hp.ops()
            xs, yz = hp.ops(("x-", "x+")), hp.ops(("y-", "y+", "z-", "z+"))
            assert sorted(xs + yz) == sorted(full)
            for sub in (xs, yz):
                sends = [f for k, f, _ in sub if k == "send"]
                recvs = [f for k, f, _ in sub if k == "recv"]
                assert sends == [f for f in FACES if f in sends]
                assert recvs == [OPPOSITE[f] for f in sends]
                # order within the subset is the order in the full exchange
                assert [full.index(o) for o in sub if o[0] == "send"] == sorted(
                    full.index(o) for o in sub if o[0] == "send")
