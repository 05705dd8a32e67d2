"""3D halo exchange plan on a periodic rank grid (config C4; SHOC-style stencil
boundaries, PAPER.md [L14:c1929 §3], generalised to 3D subarray faces;
reading A17 in DESIGN.md).

A rank owns an interior of n^3 elements inside a C-ordered local array
A[z][y][x] of (n+2h)^3 elements (ghost width h).  For each of the 6 faces it
sends its boundary layer of thickness h to the neighbour on that side and
receives the neighbour's opposite boundary layer into its ghost layer.  Each
face is one committed subarray type; the 12 transfers of one exchange go out
as one dt_group (one persistent P2P kernel, or one NCCL group per chunk).
"""
from __future__ import annotations

from dataclasses import dataclass

FACES = ("x-", "x+", "y-", "y+", "z-", "z+")
_DIM = {"z": 0, "y": 1, "x": 2}


def grid_coords(rank: int, dims=(2, 2, 2)):
    """rank -> (pz, py, px), x fastest."""
    pz, py, px = dims
    return (rank // (py * px), (rank // px) % py, rank % px)


def grid_rank(c, dims=(2, 2, 2)):
    pz, py, px = dims
    return ((c[0] % pz) * py + (c[1] % py)) * px + (c[2] % px)


def neighbour(rank: int, face: str, dims=(2, 2, 2)) -> int:
    c = list(grid_coords(rank, dims))
    c[_DIM[face[0]]] += -1 if face[1] == "-" else 1
    return grid_rank(c, dims)


def face_box(face: str, n: int, h: int, ghost: bool):
    """(subsizes, starts) of a face layer in the (n+2h)^3 array, C order [z, y, x]."""
    d = _DIM[face[0]]
    sub, st = [n, n, n], [h, h, h]
    sub[d] = h
    if face[1] == "-":
        st[d] = 0 if ghost else h
    else:
        st[d] = n + h if ghost else n
    return sub, st


OPPOSITE = {"x-": "x+", "x+": "x-", "y-": "y+", "y+": "y-", "z-": "z+", "z+": "z-"}


@dataclass
class HaloPlan:
    n: int
    h: int
    dims: tuple
    rank: int
    send_types: dict
    recv_types: dict

    def exchange(self, comm, buf, stream=None, faces=FACES):
        """Post the transfers sent through `faces` (all 12 of an exchange by
        default) as one group.  The message sent
        through face f is received by the neighbour through its face OPPOSITE[f];
        messages between the same pair are matched in posting order, so both sides
        post in one global order keyed by the SENDER's face f: sends go out in
        FACES order, and the receive matching the peer's send through f (into my
        ghost layer OPPOSITE[f], from my neighbour on that side) is posted in the
        same FACES order.  With 2 ranks per dimension both x neighbours are the
        same rank, and this ordering still pairs x- sends with x+ ghosts."""
        comm.group_start()
        for kind, face, peer in self.ops(faces):
            if kind == "send":
                comm.sendrecv(buf, 1, self.send_types[face], peer, None, 0, None, -1, stream=stream)
            else:
                comm.sendrecv(None, 0, None, -1, buf, 1, self.recv_types[face], peer, stream=stream)
        comm.group_end(stream)

    def direct_plan(self, comm, buf, group=None, single_rank=False, faces=FACES):
        """The same exchange as a persistent direct plan (dt_xplan): one kernel per
        exchange writes every boundary layer straight into the neighbour's ghost
        layer in peer memory.  Tag = index of the SENDER's face in FACES, so the
        pairing is unique even when both neighbours in a dimension are one rank."""
        from .dt import XPlan
        sends = [(buf, 1, self.send_types[f], neighbour(self.rank, f, self.dims), i)
                 for i, f in enumerate(FACES) if f in faces]
        recvs = [(buf, 1, self.recv_types[OPPOSITE[f]], neighbour(self.rank, OPPOSITE[f], self.dims), i)
                 for i, f in enumerate(FACES) if f in faces]
        if single_rank:
            return XPlan.local(comm, sends, recvs)
        return XPlan.from_process_group(comm, sends, recvs, group)

    def ops(self, faces=FACES):
        """[(kind, face, peer)] in posting order: kind 'send' (my boundary layer `face`
        to `peer`) or 'recv' (ghost layer `face` from `peer`), for the transfers
        sent through `faces`."""
        fs = [f for f in FACES if f in faces]
        out = [("send", f, neighbour(self.rank, f, self.dims)) for f in fs]
        out += [("recv", OPPOSITE[f], neighbour(self.rank, OPPOSITE[f], self.dims)) for f in fs]
        return out

    def hybrid(self, comm, buf, stream, group=None, single_rank=False):
        """Hybrid exchange: the y/z faces (long contiguous runs of n*h elements)
        go through a persistent direct plan on `stream`, the x faces (one element
        per run, 4-B blocks) through the packed ring group on a second stream, so
        the short-block faces move as dense packed fragments while the long-run
        faces skip the ring.  Returns a callable that posts one exchange, ordered
        on `stream` (the second stream joins back through an event)."""
        import torch
        yz = tuple(f for f in FACES if f[0] != "x")
        xs = tuple(f for f in FACES if f[0] == "x")
        xp = self.direct_plan(comm, buf, group=group, single_rank=single_rank, faces=yz)
        side = torch.cuda.Stream(device=stream.device)
        fork, join = torch.cuda.Event(), torch.cuda.Event()

        def run():
            fork.record(stream)
            side.wait_event(fork)
            self.exchange(comm, buf, stream=side, faces=xs)
            join.record(side)
            xp.start(stream)
            stream.wait_event(join)

        run.plan = xp
        run.check = lambda: (xp.check(), comm.check())
        return run


def make_plan(rank: int, n: int = 512, h: int = 1, dims=(2, 2, 2), basic: str = "FLOAT") -> HaloPlan:
    from .dt import Type
    L = n + 2 * h
    b = Type.basic(basic)
    st, rt = {}, {}
    for f in FACES:
        sub, s = face_box(f, n, h, ghost=False)
        st[f] = b.subarray([L, L, L], sub, s, "C").commit()
        sub, s = face_box(f, n, h, ghost=True)
        rt[f] = b.subarray([L, L, L], sub, s, "C").commit()
    return HaloPlan(n, h, tuple(dims), rank, st, rt)
