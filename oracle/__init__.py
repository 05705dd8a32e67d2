"""CPU oracle for MPI-derived-datatype pack/unpack (Wu et al., HPDC'16).

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
package.  The product (``paper_conf_hpdc_wubvjd16_b200`` / ``libdt.so``) never
imports, links or calls it, and shares no code with it.

``oracle.c`` is the plain typemap walk (PAPER.md [L16:c5201 §3.2]: pack gathers the
typemap's bytes into the contiguous buffer, unpack scatters them back;
constructors [L14:c1262 §3]; MPI-3.1 §4.1 semantics).  ``ref.py`` is an
independent pure-Python twin for tiny inputs.  This module compiles
``oracle.c`` with gcc on first use and wraps it with ctypes.

Parity status: every function here is pinned by tests/test_oracle_*.py
(closed forms, numpy slicing equivalences, the pure-Python twin, brute force,
golden typemaps in tests/golden/).  None is "parity unpinned".
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

BASIC = {"BYTE": 0, "CHAR": 1, "INT8": 2, "INT16": 3, "INT32": 4, "INT64": 5, "FLOAT": 6, "DOUBLE": 7}
BASIC_SIZE = [1, 1, 1, 2, 4, 8, 4, 8]


def build(force: bool = False) -> str:
    """Compile oracle.c -> liboracle.so (plain gcc -O2; pthreads for the timing mode)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c99", "-shared", "-fPIC", "-o", tmp, _SRC, "-lpthread"])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    with _lock:
        if _lib is None:
            L = C.CDLL(build())
            P, I64, VP = C.c_void_p, C.c_int64, C.c_void_p
            pi = C.POINTER(C.c_int64)
            sig = {
                "or_basic": (P, [C.c_int]),
                "or_contiguous": (P, [I64, P]),
                "or_vector": (P, [I64, I64, I64, P]),
                "or_hvector": (P, [I64, I64, I64, P]),
                "or_indexed": (P, [I64, pi, pi, P]),
                "or_hindexed": (P, [I64, pi, pi, P]),
                "or_indexed_block": (P, [I64, I64, pi, P]),
                "or_hindexed_block": (P, [I64, I64, pi, P]),
                "or_struct": (P, [I64, pi, pi, C.POINTER(C.c_void_p)]),
                "or_subarray": (P, [C.c_int, pi, pi, pi, C.c_int, P]),
                "or_resized": (P, [P, I64, I64]),
                "or_free": (None, [P]),
                "or_info": (None, [P, pi]),
                "or_typemap": (I64, [P, pi, pi, I64]),
                "or_pack": (I64, [P, I64, VP, VP, I64, I64]),
                "or_unpack": (I64, [P, I64, VP, VP, I64, I64]),
                "or_pack_mt": (I64, [P, I64, VP, VP, I64, I64, C.c_int]),
                "or_unpack_mt": (I64, [P, I64, VP, VP, I64, I64, C.c_int]),
                "or_addr_of": (I64, [P, I64, pi, I64, pi]),
            }
            for name, (res, args) in sig.items():
                f = getattr(L, name)
                f.restype = res
                f.argtypes = args
            _lib = L
    return _lib


def _arr(a):
    a = np.ascontiguousarray(np.asarray(a, dtype=np.int64))
    return a, a.ctypes.data_as(C.POINTER(C.c_int64))


class OType:
    """A constructor-tree type in the oracle.  Keeps its components alive."""

    def __init__(self, handle, keep=()):
        if not handle:
            raise ValueError("oracle constructor failed")
        self.h = C.c_void_p(handle)
        self._keep = keep

    def __del__(self):
        try:
            if self.h and _lib is not None:
                _lib.or_free(self.h)
        except Exception:
            pass

    # ---- constructors (MPI-3.1 §4.1; PAPER.md [L14:c1262 §3]) ----
    @staticmethod
    def basic(kind):
        k = BASIC[kind] if isinstance(kind, str) else int(kind)
        return OType(lib().or_basic(k))

    def contiguous(self, n):
        return OType(lib().or_contiguous(n, self.h), (self,))

    def vector(self, count, blocklen, stride):
        return OType(lib().or_vector(count, blocklen, stride, self.h), (self,))

    def hvector(self, count, blocklen, stride_bytes):
        return OType(lib().or_hvector(count, blocklen, stride_bytes, self.h), (self,))

    def indexed(self, blocklens, displs):
        b, pb = _arr(blocklens)
        d, pd = _arr(displs)
        assert len(b) == len(d)
        return OType(lib().or_indexed(len(b), pb, pd, self.h), (self,))

    def hindexed(self, blocklens, displs_bytes):
        b, pb = _arr(blocklens)
        d, pd = _arr(displs_bytes)
        assert len(b) == len(d)
        return OType(lib().or_hindexed(len(b), pb, pd, self.h), (self,))

    def indexed_block(self, blocklen, displs):
        d, pd = _arr(displs)
        return OType(lib().or_indexed_block(len(d), blocklen, pd, self.h), (self,))

    def hindexed_block(self, blocklen, displs_bytes):
        d, pd = _arr(displs_bytes)
        return OType(lib().or_hindexed_block(len(d), blocklen, pd, self.h), (self,))

    @staticmethod
    def struct(blocklens, displs_bytes, types):
        b, pb = _arr(blocklens)
        d, pd = _arr(displs_bytes)
        assert len(b) == len(d) == len(types)
        hs = (C.c_void_p * max(1, len(types)))(*[t.h.value for t in types])
        return OType(lib().or_struct(len(b), pb, pd, hs), tuple(types))

    def subarray(self, sizes, subsizes, starts, order="C"):
        s, ps = _arr(sizes)
        ss, pss = _arr(subsizes)
        st, pst = _arr(starts)
        o = 0 if order in ("C", 0) else 1
        return OType(lib().or_subarray(len(s), ps, pss, pst, o, self.h), (self,))

    def resized(self, lb, extent):
        return OType(lib().or_resized(self.h, lb, extent), (self,))

    # ---- queries ----
    def info(self):
        out = np.zeros(7, dtype=np.int64)
        lib().or_info(self.h, out.ctypes.data_as(C.POINTER(C.c_int64)))
        keys = ("size", "lb", "ub", "extent", "true_lb", "true_ub", "nentries")
        return {k: int(v) for k, v in zip(keys, out)}

    @property
    def size(self):
        return self.info()["size"]

    @property
    def extent(self):
        return self.info()["extent"]

    def typemap(self):
        n = self.info()["nentries"]
        k = np.zeros(max(n, 1), dtype=np.int64)
        d = np.zeros(max(n, 1), dtype=np.int64)
        lib().or_typemap(self.h, k.ctypes.data_as(C.POINTER(C.c_int64)), d.ctypes.data_as(C.POINTER(C.c_int64)), n)
        return k[:n], d[:n]


# ---- pack / unpack on host byte buffers ----
def pack(t: OType, count: int, buf: np.ndarray, origin: int = 0, pos: int = 0, length: int | None = None,
         threads: int = 1) -> np.ndarray:
    """Pack stream bytes [pos, pos+length) of `count` instances rooted at buf[origin]."""
    assert buf.dtype == np.uint8 and buf.flags.c_contiguous
    total = count * t.size
    if length is None:
        length = max(0, total - pos)
    n = max(0, min(length, total - pos))
    out = np.empty(max(n, 1), dtype=np.uint8)
    base = buf.ctypes.data + origin
    if threads > 1:
        got = lib().or_pack_mt(t.h, count, base, out.ctypes.data, pos, length, threads)
    else:
        got = lib().or_pack(t.h, count, base, out.ctypes.data, pos, length)
    assert got == n
    return out[:n]


def unpack(t: OType, count: int, packed: np.ndarray, buf: np.ndarray, origin: int = 0, pos: int = 0,
           threads: int = 1) -> int:
    """Scatter packed (stream bytes [pos, pos+len(packed))) into buf (in place)."""
    assert buf.dtype == np.uint8 and buf.flags.c_contiguous and packed.dtype == np.uint8
    packed = np.ascontiguousarray(packed)
    base = buf.ctypes.data + origin
    if threads > 1:
        return lib().or_unpack_mt(t.h, count, packed.ctypes.data, base, pos, len(packed), threads)
    return lib().or_unpack(t.h, count, packed.ctypes.data, base, pos, len(packed))


def addr_of(t: OType, count: int, positions) -> np.ndarray:
    """Byte address (relative to the origin) of each stream byte position (sorted ascending)."""
    p, pp = _arr(positions)
    assert np.all(np.diff(p) >= 0)
    out = np.zeros(max(len(p), 1), dtype=np.int64)
    lib().or_addr_of(t.h, count, pp, len(p), out.ctypes.data_as(C.POINTER(C.c_int64)))
    return out[: len(p)]


def sendrecv(stype: OType, scount: int, sbuf: np.ndarray, rtype: OType, rcount: int, rbuf: np.ndarray,
             sorigin: int = 0, rorigin: int = 0) -> None:
    """rbuf' = unpack(rtype, rcount, pack(stype, scount, sbuf)) over the
    first scount*size(stype) bytes; truncation (send > recv) is an error (reading A12)."""
    n = scount * stype.size
    if n > rcount * rtype.size:
        raise ValueError("truncate")
    p = pack(stype, scount, sbuf, sorigin)
    unpack(rtype, rcount, p, rbuf, rorigin)


def from_recipe(r) -> OType:
    """Build an oracle type from a workloads/ recipe tuple (constructor name first)."""
    op = r[0]
    if op == "basic":
        return OType.basic(r[1])
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
        return OType.struct(r[1], r[2], [from_recipe(x) for x in r[3]])
    if op == "subarray":
        return from_recipe(r[5]).subarray(r[1], r[2], r[3], r[4])
    if op == "resized":
        return from_recipe(r[1]).resized(r[2], r[3])
    raise ValueError(f"unknown recipe op {op!r}")
