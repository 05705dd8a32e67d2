"""Thin ctypes binding over libdt.so (include/dt.h).  Argument marshalling only:
every byte of pack/unpack/sendrecv moves inside the library's CUDA kernels.

torch is used only as the plumbing for device memory and streams: tensors are
passed as ``data_ptr()`` integers and streams as ``cuda_stream`` handles.  There
is no CPU fallback: if libdt.so is missing or a GPU is absent, calls fail loudly.
"""
from __future__ import annotations

import ctypes as C
import os
import threading

from . import _build

_lock = threading.Lock()
_lib = None

STATUS = {0: "DT_OK", 1: "DT_ERR_ARG", 2: "DT_ERR_NOT_COMMITTED", 3: "DT_ERR_OVERLAP", 4: "DT_ERR_TRUNCATE",
          5: "DT_ERR_CUDA", 6: "DT_ERR_NCCL", 7: "DT_ERR_NOMEM", 8: "DT_ERR_TIMEOUT", 9: "DT_ERR_UNSUPPORTED"}
BASIC = {"BYTE": 0, "CHAR": 1, "INT8": 2, "INT16": 3, "INT32": 4, "INT64": 5, "FLOAT": 6, "DOUBLE": 7}
XFER_P2P, XFER_NCCL, XFER_CE = 0, 1, 2


class DTError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status
        self.name = STATUS.get(status, str(status))


class FormInfo(C.Structure):
    _fields_ = [("size", C.c_int64), ("lb", C.c_int64), ("extent", C.c_int64), ("true_lb", C.c_int64),
                ("true_extent", C.c_int64), ("nblocks", C.c_int64), ("tsize", C.c_int64),
                ("nlevels", C.c_int32), ("level_is_list", C.c_int32 * 8), ("level_count", C.c_int64 * 8),
                ("level_stride", C.c_int64 * 8), ("granularity", C.c_int64)]


class XOp(C.Structure):
    _fields_ = [("buf", C.c_void_p), ("count", C.c_int64), ("type", C.c_void_p), ("peer", C.c_int32),
                ("tag", C.c_int32)]


class XferOpts(C.Structure):
    _fields_ = [("chunk_bytes", C.c_int64), ("depth", C.c_int32), ("mode", C.c_int32), ("ctas", C.c_int32),
                ("flags", C.c_int32)]


P = C.c_void_p
I64 = C.c_int64
PI64 = C.POINTER(C.c_int64)
_SIGS = {
    "dt_basic_type": (P, [C.c_int]),
    "dt_create_contiguous": (C.c_int, [I64, P, C.POINTER(P)]),
    "dt_create_vector": (C.c_int, [I64, I64, I64, P, C.POINTER(P)]),
    "dt_create_hvector": (C.c_int, [I64, I64, I64, P, C.POINTER(P)]),
    "dt_create_indexed": (C.c_int, [I64, PI64, PI64, P, C.POINTER(P)]),
    "dt_create_hindexed": (C.c_int, [I64, PI64, PI64, P, C.POINTER(P)]),
    "dt_create_indexed_block": (C.c_int, [I64, I64, PI64, P, C.POINTER(P)]),
    "dt_create_hindexed_block": (C.c_int, [I64, I64, PI64, P, C.POINTER(P)]),
    "dt_create_struct": (C.c_int, [I64, PI64, PI64, C.POINTER(P), C.POINTER(P)]),
    "dt_create_subarray": (C.c_int, [C.c_int, PI64, PI64, PI64, C.c_int, P, C.POINTER(P)]),
    "dt_create_resized": (C.c_int, [P, I64, I64, C.POINTER(P)]),
    "dt_commit": (C.c_int, [P]),
    "dt_get_size": (C.c_int, [P, PI64]),
    "dt_get_extent": (C.c_int, [P, PI64, PI64]),
    "dt_get_true_extent": (C.c_int, [P, PI64, PI64]),
    "dt_free": (C.c_int, [C.POINTER(P)]),
    "dt_pack": (C.c_int, [P, I64, P, P, I64, PI64, P]),
    "dt_unpack": (C.c_int, [P, I64, P, P, I64, PI64, P]),
    "dt_pack_host": (C.c_int, [P, I64, P, P, I64, PI64, P]),
    "dt_copy": (C.c_int, [P, I64, P, P, I64, P, P]),
    "dt_unpack_host": (C.c_int, [P, I64, P, P, I64, PI64, P]),
    "dt_get_form": (C.c_int, [P, C.POINTER(FormInfo)]),
    "dt_flatten": (C.c_int, [P, I64, PI64, PI64, I64, PI64]),
    "dt_plan": (C.c_int, [P, I64, C.c_uint64, C.c_uint64, I64, I64, C.POINTER(C.c_int), PI64]),
    "dt_comm_init": (C.c_int, [C.c_int, C.c_int, P, C.c_int, C.POINTER(XferOpts), C.POINTER(P)]),
    "dt_nccl_unique_id": (C.c_int, [P]),
    "dt_comm_local_handle": (C.c_int, [P, P, C.POINTER(C.c_size_t)]),
    "dt_comm_connect": (C.c_int, [P, P, C.c_size_t]),
    "dt_sendrecv": (C.c_int, [P, I64, P, C.c_int, P, I64, P, C.c_int, P, C.POINTER(XferOpts), P]),
    "dt_group_start": (C.c_int, [P]),
    "dt_group_end": (C.c_int, [P, P]),
    "dt_comm_check": (C.c_int, [P]),
    "dt_comm_free": (C.c_int, [C.POINTER(P)]),
    "dt_type_serialize": (C.c_int, [P, P, C.POINTER(C.c_size_t)]),
    "dt_type_deserialize": (C.c_int, [P, C.c_size_t, C.POINTER(P)]),
    "dt_xplan_create": (C.c_int, [P, C.c_int, P, C.c_int, P, C.POINTER(P)]),
    "dt_xplan_local_blob": (C.c_int, [P, P, C.POINTER(C.c_size_t)]),
    "dt_xplan_connect": (C.c_int, [P, P, C.POINTER(C.c_size_t)]),
    "dt_xplan_start": (C.c_int, [P, P]),
    "dt_xplan_check": (C.c_int, [P]),
    "dt_xplan_free": (C.c_int, [C.POINTER(P)]),
    "dt_last_error": (C.c_char_p, []),
    "dt_version": (C.c_char_p, []),
}


def lib_path() -> str:
    return _build.LIB


def lib():
    """Load libdt.so (building it in-tree with nvcc first if it is stale)."""
    global _lib
    with _lock:
        if _lib is None:
            if _build.needs_build():
                _build.build()
            L = C.CDLL(_build.LIB)
            for name, (res, args) in _SIGS.items():
                f = getattr(L, name)
                f.restype = res
                f.argtypes = args
            _lib = L
    return _lib


def _check(st):
    if st != 0:
        msg = lib().dt_last_error()
        raise DTError(st, msg.decode() if msg else "")


def _i64(a):
    import numpy as np
    a = np.ascontiguousarray(np.asarray(a, dtype=np.int64))
    return a, a.ctypes.data_as(PI64)


class Type:
    """A datatype handle (MPI-3.1 §4.1 constructors; PAPER.md [L14:c1262 §3])."""

    def __init__(self, handle, predefined=False, keep=()):
        if not handle:
            raise DTError(1, lib().dt_last_error().decode())
        self.h = P(handle) if not isinstance(handle, P) else handle
        self.predefined = predefined
        self._keep = keep

    def __del__(self):
        try:
            if not self.predefined and self.h and _lib is not None:
                _lib.dt_free(C.byref(self.h))
        except Exception:
            pass

    @staticmethod
    def basic(kind):
        k = BASIC[kind] if isinstance(kind, str) else int(kind)
        return Type(lib().dt_basic_type(k), predefined=True)

    def _new(self, fn, *args, keep=None):
        out = P()
        _check(fn(*args, C.byref(out)))
        return Type(out, keep=keep if keep is not None else (self,))

    def contiguous(self, n):
        return self._new(lib().dt_create_contiguous, n, self.h)

    def vector(self, count, blocklen, stride):
        return self._new(lib().dt_create_vector, count, blocklen, stride, self.h)

    def hvector(self, count, blocklen, stride_bytes):
        return self._new(lib().dt_create_hvector, count, blocklen, stride_bytes, self.h)

    def indexed(self, blocklens, displs):
        b, pb = _i64(blocklens)
        d, pd = _i64(displs)
        return self._new(lib().dt_create_indexed, len(b), pb, pd, self.h)

    def hindexed(self, blocklens, displs_bytes):
        b, pb = _i64(blocklens)
        d, pd = _i64(displs_bytes)
        return self._new(lib().dt_create_hindexed, len(b), pb, pd, self.h)

    def indexed_block(self, blocklen, displs):
        d, pd = _i64(displs)
        return self._new(lib().dt_create_indexed_block, len(d), blocklen, pd, self.h)

    def hindexed_block(self, blocklen, displs_bytes):
        d, pd = _i64(displs_bytes)
        return self._new(lib().dt_create_hindexed_block, len(d), blocklen, pd, self.h)

    @staticmethod
    def struct(blocklens, displs_bytes, types):
        b, pb = _i64(blocklens)
        d, pd = _i64(displs_bytes)
        hs = (P * max(1, len(types)))(*[t.h.value for t in types])
        out = P()
        _check(lib().dt_create_struct(len(b), pb, pd, hs, C.byref(out)))
        return Type(out, keep=tuple(types))

    def subarray(self, sizes, subsizes, starts, order="C"):
        s, ps = _i64(sizes)
        ss, pss = _i64(subsizes)
        st, pst = _i64(starts)
        o = 0 if order in ("C", 0) else 1
        return self._new(lib().dt_create_subarray, len(s), ps, pss, pst, o, self.h)

    def resized(self, lb, extent):
        return self._new(lib().dt_create_resized, self.h, lb, extent)

    def commit(self):
        _check(lib().dt_commit(self.h))
        return self

    @property
    def size(self):
        v = I64()
        _check(lib().dt_get_size(self.h, C.byref(v)))
        return v.value

    @property
    def lb(self):
        a, b = I64(), I64()
        _check(lib().dt_get_extent(self.h, C.byref(a), C.byref(b)))
        return a.value

    @property
    def extent(self):
        a, b = I64(), I64()
        _check(lib().dt_get_extent(self.h, C.byref(a), C.byref(b)))
        return b.value

    @property
    def true_extent(self):
        a, b = I64(), I64()
        _check(lib().dt_get_true_extent(self.h, C.byref(a), C.byref(b)))
        return a.value, b.value

    def form(self):
        fi = FormInfo()
        _check(lib().dt_get_form(self.h, C.byref(fi)))
        return fi

    def flatten(self, count=1):
        import numpy as np
        n = I64()
        _check(lib().dt_flatten(self.h, count, None, None, 0, C.byref(n)))
        d = np.zeros(max(1, n.value), dtype=np.int64)
        ln = np.zeros(max(1, n.value), dtype=np.int64)
        _check(lib().dt_flatten(self.h, count, d.ctypes.data_as(PI64), ln.ctypes.data_as(PI64), n.value,
                                C.byref(n)))
        return d[: n.value], ln[: n.value]

    def serialize(self) -> bytes:
        """dt_type_serialize: the flattened form + bounds, to ship to another rank."""
        n = C.c_size_t(0)
        _check(lib().dt_type_serialize(self.h, None, C.byref(n)))
        buf = C.create_string_buffer(n.value)
        _check(lib().dt_type_serialize(self.h, buf, C.byref(n)))
        return buf.raw[: n.value]

    @staticmethod
    def deserialize(blob: bytes) -> "Type":
        """dt_type_deserialize: a new (uncommitted) handle with the serialized typemap."""
        h = P()
        buf = C.create_string_buffer(blob, len(blob))
        _check(lib().dt_type_deserialize(buf, len(blob), C.byref(h)))
        return Type(h)

    def plan(self, count, origin_addr, packed_addr, pos, nbytes):
        k = C.c_int()
        g = I64()
        _check(lib().dt_plan(self.h, count, origin_addr, packed_addr, pos, nbytes, C.byref(k), C.byref(g)))
        return k.value, g.value


def from_recipe(r) -> Type:
    """Build a library type from a workloads/ recipe tuple (constructor name first)."""
    op = r[0]
    if op == "basic":
        return Type.basic(r[1])
    if op == "contiguous":
        return from_recipe(r[2]).contiguous(r[1])
    if op == "vector":
        return from_recipe(r[4]).vector(r[1], r[2], r[3])
    if op == "hvector":
        return from_recipe(r[4]).hvector(r[1], r[2], r[3])
    if op == "indexed":
        return from_recipe(r[3]).indexed(r[1], r[2])
    if op == "hindexed":
        return from_recipe(r[3]).hindexed(r[1], r[2])
    if op == "indexed_block":
        return from_recipe(r[3]).indexed_block(r[1], r[2])
    if op == "hindexed_block":
        return from_recipe(r[3]).hindexed_block(r[1], r[2])
    if op == "struct":
        return Type.struct(r[1], r[2], [from_recipe(x) for x in r[3]])
    if op == "subarray":
        return from_recipe(r[5]).subarray(r[1], r[2], r[3], r[4])
    if op == "resized":
        return from_recipe(r[1]).resized(r[2], r[3])
    raise ValueError(f"unknown recipe op {op!r}")


def _ptr(x):
    if isinstance(x, int):
        return x
    return x.data_ptr()


def _stream(stream):
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


def pack(t: Type, count: int, origin, packed, pos: int = 0, nbytes: int | None = None, stream=None,
         origin_offset: int = 0) -> int:
    """dt_pack: stream bytes [pos, pos+nbytes) of `count` instances rooted at
    origin (+origin_offset bytes) into `packed`.  Returns bytes packed."""
    n = I64((count * t.size - pos) if nbytes is None else nbytes)
    _check(lib().dt_pack(t.h, count, _ptr(origin) + origin_offset, _ptr(packed), pos, C.byref(n), _stream(stream)))
    return n.value


def unpack(t: Type, count: int, packed, origin, pos: int = 0, nbytes: int | None = None, stream=None,
           origin_offset: int = 0) -> int:
    """dt_unpack: scatter `packed` (stream bytes [pos, pos+nbytes)) to the layout at origin."""
    n = I64((count * t.size - pos) if nbytes is None else nbytes)
    _check(lib().dt_unpack(t.h, count, _ptr(packed), _ptr(origin) + origin_offset, pos, C.byref(n),
                           _stream(stream)))
    return n.value


def pack_host(t: Type, count: int, origin_addr: int, packed_addr: int, pos: int = 0, nbytes: int | None = None,
              stream=None) -> int:
    n = I64((count * t.size - pos) if nbytes is None else nbytes)
    _check(lib().dt_pack_host(t.h, count, origin_addr, packed_addr, pos, C.byref(n), _stream(stream)))
    return n.value


def unpack_host(t: Type, count: int, packed_addr: int, origin_addr: int, pos: int = 0, nbytes: int | None = None,
                stream=None) -> int:
    n = I64((count * t.size - pos) if nbytes is None else nbytes)
    _check(lib().dt_unpack_host(t.h, count, packed_addr, origin_addr, pos, C.byref(n), _stream(stream)))
    return n.value


# ------------------------------------------------------------------ GPU <-> GPU transfer
def exchange_blobs(blob: bytes, group=None) -> bytes:
    """All-gather one equal-size byte blob per rank (rank-major concatenation)
    through torch.distributed — plumbing for dt_comm_connect's IPC handles."""
    import torch.distributed as tdist
    ws = tdist.get_world_size(group)
    out = [None] * ws
    tdist.all_gather_object(out, blob, group=group)
    assert all(len(b) == len(blob) for b in out), "handle blobs differ in size"
    return b"".join(out)


def broadcast_id(idbytes, group=None) -> bytes:
    """Broadcast rank 0's 128-byte NCCL unique id."""
    import torch.distributed as tdist
    obj = [idbytes]
    tdist.broadcast_object_list(obj, src=0, group=group)
    return obj[0]


class Comm:
    """dt_comm_t: this rank's endpoint (receive rings + flags, or a NCCL communicator)."""

    def __init__(self, rank: int, nranks: int, device: int, chunk_bytes: int = 1 << 20, depth: int = 0,
                 mode: int = XFER_P2P, ctas: int = 0, nccl_id: bytes | None = None, ring_loopback: bool = False):
        # ring_loopback: send-to-self goes through the ring pipeline instead of the fused dt_copy
        self.opts = XferOpts(chunk_bytes, depth, mode, ctas, 1 if ring_loopback else 0)
        self.h = P()
        self.rank, self.nranks = rank, nranks
        idbuf = C.create_string_buffer(nccl_id, 128) if nccl_id else None
        _check(lib().dt_comm_init(rank, nranks, idbuf, device, C.byref(self.opts), C.byref(self.h)))

    @staticmethod
    def nccl_unique_id() -> bytes:
        buf = C.create_string_buffer(128)
        _check(lib().dt_nccl_unique_id(buf))
        return buf.raw

    @classmethod
    def from_process_group(cls, group=None, device: int | None = None, **opts):
        """Create the endpoint on every rank of `group` and connect the ring mappings
        (IPC handles all-gathered once, [L20:c3123], [L20:c3807])."""
        import torch
        import torch.distributed as tdist
        rank, ws = tdist.get_rank(group), tdist.get_world_size(group)
        if device is None:
            device = torch.cuda.current_device()
        nid = None
        if opts.get("mode", XFER_P2P) == XFER_NCCL:
            nid = broadcast_id(cls.nccl_unique_id() if rank == 0 else None, group)
        c = cls(rank, ws, device, nccl_id=nid, **opts)
        c.connect(exchange_blobs(c.local_handle(), group))
        return c

    def local_handle(self) -> bytes:
        n = C.c_size_t(0)
        _check(lib().dt_comm_local_handle(self.h, None, C.byref(n)))
        buf = C.create_string_buffer(n.value)
        _check(lib().dt_comm_local_handle(self.h, buf, C.byref(n)))
        return buf.raw[: n.value]

    def connect(self, all_handles: bytes):
        per = len(all_handles) // self.nranks
        buf = C.create_string_buffer(all_handles, len(all_handles))
        _check(lib().dt_comm_connect(self.h, buf, per))

    def sendrecv(self, sbuf, scount, stype, dest, rbuf, rcount, rtype, source, stream=None, sbuf_offset=0,
                 rbuf_offset=0):
        sp = (_ptr(sbuf) + sbuf_offset) if sbuf is not None else None
        rp = (_ptr(rbuf) + rbuf_offset) if rbuf is not None else None
        _check(lib().dt_sendrecv(sp, scount, stype.h if stype else None, dest, rp, rcount,
                                 rtype.h if rtype else None, source, self.h, None, _stream(stream)))

    def group_start(self):
        _check(lib().dt_group_start(self.h))

    def group_end(self, stream=None):
        _check(lib().dt_group_end(self.h, _stream(stream)))

    def check(self):
        _check(lib().dt_comm_check(self.h))

    def free(self):
        if self.h:
            _check(lib().dt_comm_free(C.byref(self.h)))
            self.h = P()

    def __del__(self):
        try:
            if self.h and _lib is not None:
                _lib.dt_comm_free(C.byref(self.h))
        except Exception:
            pass


def copy(stype: Type, scount: int, src, rtype: Type, rcount: int, dst, stream=None, src_offset: int = 0,
         dst_offset: int = 0) -> None:
    """dt_copy: fused datatype -> datatype copy on one GPU (no packed buffer)."""
    _check(lib().dt_copy(stype.h, scount, _ptr(src) + src_offset, rtype.h, rcount, _ptr(dst) + dst_offset,
                         _stream(stream)))


# ------------------------------------------------------------------ persistent direct exchange (f1 across GPUs)
class XPlan:
    """dt_xplan_t: a fixed set of sends and receives executed as ONE kernel per rank
    per start: each send is copied from its local layout straight into the
    receiver's layout in peer memory (NVLink / CUDA IPC), no ring and no unpack.

    sends / recvs: lists of (buf, count, type, peer, tag) (buf: tensor or device
    address; tag pairs a send of rank r to rank d with d's receive from r).
    Connect with `from_process_group` (blobs all-gathered through
    torch.distributed) or, on a single rank, `local()`."""

    def __init__(self, comm: Comm, sends, recvs):
        self.comm = comm
        self._keep = (sends, recvs)
        mk = lambda ops: (XOp * max(1, len(ops)))(*[XOp(_ptr(b), c, t.h, p, g) for (b, c, t, p, g) in ops])  # noqa
        so, ro = mk(sends), mk(recvs)
        self.h = P()
        _check(lib().dt_xplan_create(comm.h, len(sends), so, len(recvs), ro, C.byref(self.h)))

    def local_blob(self) -> bytes:
        n = C.c_size_t(0)
        _check(lib().dt_xplan_local_blob(self.h, None, C.byref(n)))
        buf = C.create_string_buffer(n.value)
        _check(lib().dt_xplan_local_blob(self.h, buf, C.byref(n)))
        return buf.raw[: n.value]

    def connect(self, blobs):
        sizes = (C.c_size_t * len(blobs))(*[len(b) for b in blobs])
        allb = b"".join(blobs)
        buf = C.create_string_buffer(allb, max(1, len(allb)))
        _check(lib().dt_xplan_connect(self.h, buf, sizes))
        return self

    @classmethod
    def from_process_group(cls, comm: Comm, sends, recvs, group=None) -> "XPlan":
        import torch.distributed as tdist
        x = cls(comm, sends, recvs)
        out = [None] * tdist.get_world_size(group)
        tdist.all_gather_object(out, x.local_blob(), group=group)
        return x.connect(out)

    @classmethod
    def local(cls, comm: Comm, sends, recvs) -> "XPlan":
        """Single-rank plan (every peer is this rank)."""
        x = cls(comm, sends, recvs)
        return x.connect([x.local_blob()])

    def start(self, stream=None):
        _check(lib().dt_xplan_start(self.h, _stream(stream)))

    def check(self):
        _check(lib().dt_xplan_check(self.h))

    def free(self):
        if self.h:
            _check(lib().dt_xplan_free(C.byref(self.h)))
            self.h = P()

    def __del__(self):
        try:
            if self.h and _lib is not None:
                _lib.dt_xplan_free(C.byref(self.h))
        except Exception:
            pass
