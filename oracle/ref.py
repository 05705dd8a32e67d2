"""Pure-Python twin of the oracle, for tiny inputs only.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).  Written independently of
oracle.c: where oracle.c runs the constructor loops lazily over a tree, this
module materialises the explicit MPI typemap — a Python list of
``(kind, disp)`` pairs plus the pseudo-entries ``("LB", d)``, ``("UB", d)``
(explicit markers set by resized/subarray, MPI-3.1 §4.1.7) and ``("PAD", d)``
(the upper end of a struct's alignment padding, reading R-eps) — and derives
every bound from that explicit list, the way MPI-3.1 §4.1.6 states it:

    lb = min(LB markers) if any, else min(data disps)
    ub = max(UB markers) if any, else max(data end, PAD) (struct: rounded up to
         a multiple of the largest basic alignment)

Pack = concatenation over instances k < count of the bytes of each data entry
at k*extent + disp, in typemap order (PAPER.md [L16:c5201 §3.2]).
"""
from __future__ import annotations

SIZES = {0: 1, 1: 1, 2: 1, 3: 2, 4: 4, 5: 8, 6: 4, 7: 8}


class RType:
    def __init__(self, tmap, is_struct=False):
        self.tmap = tmap  # list of (kind|'LB'|'UB'|'PAD', disp)
        data = [(k, d) for k, d in tmap if isinstance(k, int)]
        lbs = [d for k, d in tmap if k == "LB"]
        ubs = [d for k, d in tmap if k == "UB"]
        pads = [d for k, d in tmap if k == "PAD"]
        self.entries = data
        self.size = sum(SIZES[k] for k, _ in data)
        self.align = max([SIZES[k] for k, _ in data], default=1)
        if data:
            self.true_lb = min(d for _, d in data)
            self.true_ub = max(d + SIZES[k] for k, d in data)
        else:
            self.true_lb = self.true_ub = 0
        self.lb = min(lbs) if lbs else (self.true_lb if data else 0)
        if ubs:
            self.ub = max(ubs)
        elif data:
            self.ub = max([self.true_ub] + pads)
            if is_struct:
                e = self.ub - self.lb
                self.ub += (-e) % self.align
                # the padding end becomes sticky for copies of this struct
                self.tmap = [x for x in self.tmap if x[0] != "PAD"] + [("PAD", self.ub)]
        else:
            self.ub = 0

    @property
    def extent(self):
        return self.ub - self.lb

    def shifted(self, s):
        return [(k, d + s) for k, d in self.tmap]


def basic(kind):
    return RType([(kind, 0)])


def _copies(pairs):
    out = []
    for t, s in pairs:
        out += t.shifted(s)
    return out


def contiguous(n, t):
    return RType(_copies([(t, i * t.extent) for i in range(n)]))


def hvector(c, b, s, t):
    return RType(_copies([(t, i * s + j * t.extent) for i in range(c) for j in range(b)]))


def vector(c, b, s, t):
    return hvector(c, b, s * t.extent, t)


def hindexed(B, D, t):
    return RType(_copies([(t, D[i] + j * t.extent) for i in range(len(B)) for j in range(B[i])]))


def indexed(B, D, t):
    return hindexed(B, [d * t.extent for d in D], t)


def hindexed_block(b, D, t):
    return hindexed([b] * len(D), D, t)


def indexed_block(b, D, t):
    return indexed([b] * len(D), D, t)


def struct(B, D, T):
    return RType(_copies([(T[i], D[i] + j * T[i].extent) for i in range(len(B)) for j in range(B[i])]),
                 is_struct=True)


def subarray(sizes, subsizes, starts, order, t):
    import itertools
    n = len(sizes)
    dims = list(range(n)) if order == "C" else list(range(n))[::-1]  # slowest .. fastest
    pairs = []
    for idx in itertools.product(*[range(subsizes[d]) for d in dims]):
        full = [0] * n
        for d, i in zip(dims, idx):
            full[d] = starts[d] + i
        lin = 0
        for d in dims:  # row-major over the slowest..fastest order
            lin = lin * sizes[d] + full[d]
        pairs.append((t, lin * t.extent))
    tot = 1
    for s in sizes:
        tot *= s
    body = [x for x in _copies(pairs) if x[0] not in ("LB", "UB")]
    return RType(body + [("LB", 0), ("UB", tot * t.extent)])


def resized(t, lb, extent):
    body = [x for x in t.tmap if x[0] not in ("LB", "UB", "PAD")]
    return RType(body + [("LB", lb), ("UB", lb + extent)])


def pack(t, count, buf: bytes, origin=0, pos=0, length=None):
    stream = bytearray()
    for k in range(count):
        for kind, d in t.entries:
            a = origin + k * t.extent + d
            stream += buf[a:a + SIZES[kind]]
    total = len(stream)
    if length is None:
        length = total - pos
    return bytes(stream[pos:pos + max(0, length)])


def unpack(t, count, packed: bytes, buf: bytearray, origin=0, pos=0):
    addrs = []
    for k in range(count):
        for kind, d in t.entries:
            a = origin + k * t.extent + d
            addrs += list(range(a, a + SIZES[kind]))
    for i, b in enumerate(packed):
        buf[addrs[pos + i]] = b
    return buf


def from_recipe(r):
    """Build a twin type from a workloads/ recipe tuple."""
    from oracle import BASIC
    op = r[0]
    if op == "basic":
        return basic(BASIC[r[1]])
    if op == "contiguous":
        return contiguous(r[1], from_recipe(r[2]))
    if op == "vector":
        return vector(r[1], r[2], r[3], from_recipe(r[4]))
    if op == "hvector":
        return hvector(r[1], r[2], r[3], from_recipe(r[4]))
    if op == "indexed":
        return indexed(list(r[1]), list(r[2]), from_recipe(r[3]))
    if op == "hindexed":
        return hindexed(list(r[1]), list(r[2]), from_recipe(r[3]))
    if op == "indexed_block":
        return indexed_block(r[1], list(r[2]), from_recipe(r[3]))
    if op == "hindexed_block":
        return hindexed_block(r[1], list(r[2]), from_recipe(r[3]))
    if op == "struct":
        return struct(list(r[1]), list(r[2]), [from_recipe(x) for x in r[3]])
    if op == "subarray":
        return subarray(list(r[1]), list(r[2]), list(r[3]), r[4], from_recipe(r[5]))
    if op == "resized":
        return resized(from_recipe(r[1]), r[2], r[3])
    raise ValueError(op)
