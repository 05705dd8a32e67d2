"""Pins for the CPU oracle (T0).  Each check compares the oracle with something
other than itself: hand-derived typemaps (tests/golden/), closed forms, numpy
slicing as an independent library routine, the independently written pure-Python
twin (oracle/ref.py), brute-force enumeration and address-encoding sources.

Paper passages: constructors [L14:c1262 §3]; V and T workloads [L22:c1966],
[L22:c2839 §5.1]; pack into / unpack from the contiguous buffer [L16:c5201 §3.2].
"""
import itertools
import json
import os

import numpy as np
import pytest

import oracle
from oracle import ref
from workloads import (address_words, c1_submatrix, c2_lower_triangle, c3_block_cyclic, c4_face,
                       c5_particles, fill_bytes, poison, stair_triangle, upper_triangle, PARTICLE)

HERE = os.path.dirname(os.path.abspath(__file__))
GOLD = json.load(open(os.path.join(HERE, "golden", "typemaps.json")))


def _tolist(x):
    return [_tolist(v) for v in x] if isinstance(x, (list, tuple)) else x


@pytest.mark.parametrize("case", GOLD["cases"], ids=[c["name"] for c in GOLD["cases"]])
def test_golden_typemaps(case):
    r = case["recipe"]
    for t in (oracle.from_recipe(r),):
        info = t.info()
        for k in ("size", "lb", "ub", "extent", "true_lb", "true_ub"):
            assert info[k] == case[k], (k, info[k], case[k])
        _, d = t.typemap()
        assert list(d) == case["disps"]
    tw = ref.from_recipe(r)
    assert [d for _, d in tw.entries] == case["disps"]
    for k in ("size", "lb", "ub", "extent", "true_lb", "true_ub"):
        assert getattr(tw, k) == case[k], (k,)


# ---------------------------------------------------------------- closed forms
@pytest.mark.parametrize("kind,e", [("INT32", 4), ("DOUBLE", 8), ("INT16", 2), ("BYTE", 1)])
def test_vector_closed_form(kind, e):
    """vector(c,b,s): size c*b*e; extent ((c-1)*s+b)*e for s>=b>0, c>=1."""
    b0 = oracle.OType.basic(kind)
    for c in range(1, 6):
        for b in range(1, 4):
            for s in range(b, b + 4):
                t = b0.vector(c, b, s)
                i = t.info()
                assert i["size"] == c * b * e
                assert i["extent"] == ((c - 1) * s + b) * e
                assert i["lb"] == 0 and i["true_ub"] == ((c - 1) * s + b) * e
                # packed byte p <-> source byte (p div (b e)) s e + (p mod (b e))
                _, d = t.typemap()
                p = np.arange(c * b) * e
                assert np.array_equal(d, (p // (b * e)) * s * e + (p % (b * e)))


def test_contiguous_indexed_closed_form():
    t = oracle.OType.basic("DOUBLE")
    assert t.contiguous(7).info()["size"] == 56 and t.contiguous(7).extent == 56
    B, Dd = [2, 0, 3, 1], [5, 1, 9, 0]
    i = t.indexed(B, Dd).info()
    assert i["size"] == sum(B) * 8
    nz = [k for k in range(4) if B[k] > 0]
    assert i["true_lb"] == min(Dd[k] for k in nz) * 8
    assert i["true_ub"] == max(Dd[k] + B[k] for k in nz) * 8


@pytest.mark.parametrize("n", [1, 2, 3, 17, 64])
def test_triangle_closed_form(n):
    r, _, _ = c2_lower_triangle(n)
    i = oracle.from_recipe(r).info()
    assert i["size"] == n * (n + 1) // 2 * 8            # "half the size" [L24:c3145]
    assert i["extent"] == n * n * 8 and i["lb"] == 0


def test_subarray_closed_form():
    b = oracle.OType.basic("FLOAT")
    for sizes, subs, starts in [([6, 7, 5], [2, 3, 4], [1, 2, 0]), ([3], [2], [1]), ([4, 4], [4, 1], [0, 3])]:
        for order in ("C", "F"):
            i = b.subarray(sizes, subs, starts, order).info()
            assert i["size"] == int(np.prod(subs)) * 4
            assert i["extent"] == int(np.prod(sizes)) * 4 and i["lb"] == 0


# ---------------------------------------------------------------- numpy equivalence
def test_submatrix_numpy():
    """V ([L22:c1966]): pack == column-major slice A[r0:r0+m, c0:c0+n] raveled in F order."""
    for (m, lda, r0, c0) in [(16, 40, 0, 0), (16, 40, 1, 1), (7, 13, 3, 2)]:
        rec, org, nbytes = c1_submatrix(m, lda, r0, c0)
        buf = fill_bytes(nbytes, 7)
        A = buf.view(np.float64).reshape(lda, lda).T     # A[r, c] column-major
        exp = np.ascontiguousarray(A[r0:r0 + m, c0:c0 + m].ravel(order="F")).view(np.uint8)
        got = oracle.pack(oracle.from_recipe(rec), 1, buf, org)
        assert np.array_equal(got, exp)


@pytest.mark.parametrize("n", [1, 5, 33, 128])
def test_triangle_numpy(n):
    """T ([L22:c2839]): with M = buf.reshape(n,n) (M[c,r] = A[r,c]) pack == M[triu_indices(n)]."""
    rec, _, nbytes = c2_lower_triangle(n)
    buf = fill_bytes(nbytes, 11)
    M = buf.view(np.float64).reshape(n, n)
    exp = np.ascontiguousarray(M[np.triu_indices(n)]).view(np.uint8)
    assert np.array_equal(oracle.pack(oracle.from_recipe(rec), 1, buf), exp)
    rec, _, _ = upper_triangle(n)
    exp = np.ascontiguousarray(M[np.tril_indices(n)]).view(np.uint8)
    assert np.array_equal(oracle.pack(oracle.from_recipe(rec), 1, buf), exp)


def test_stair_numpy():
    n, nb = 16, 4
    rec, _, nbytes = stair_triangle(n, nb)
    buf = fill_bytes(nbytes, 3)
    A = buf.view(np.float64).reshape(n, n).T
    exp = np.concatenate([A[nb * (j // nb):, j] for j in range(n)]).view(np.uint8)
    assert np.array_equal(oracle.pack(oracle.from_recipe(rec), 1, buf), exp)


@pytest.mark.parametrize("order", ["C", "F"])
def test_subarray_numpy(order):
    sizes, subs, starts = [6, 7, 5], [2, 3, 4], [3, 2, 1]
    buf = fill_bytes(int(np.prod(sizes)) * 4, 5)
    A = buf.view(np.uint32).reshape(sizes, order=order)
    sl = tuple(slice(s, s + n) for s, n in zip(starts, subs))
    exp = np.ascontiguousarray(A[sl].ravel(order=order)).view(np.uint8)
    t = oracle.OType.basic("INT32").subarray(sizes, subs, starts, order)
    assert np.array_equal(oracle.pack(t, 1, buf), exp)


def test_halo_face_numpy():
    n, h = 6, 1
    L = n + 2 * h
    buf = fill_bytes(L ** 3 * 4, 9)
    A = buf.view(np.uint32).reshape(L, L, L)
    for face in ("x-", "x+", "y-", "y+", "z-", "z+"):
        for ghost in (False, True):
            rec, _, _ = c4_face(face, n, h, ghost)
            st, sub = rec[3], rec[2]
            sl = tuple(slice(s, s + k) for s, k in zip(st, sub))
            exp = np.ascontiguousarray(A[sl]).ravel().view(np.uint8)
            assert np.array_equal(oracle.pack(oracle.from_recipe(rec), 1, buf), exp)


def test_hvector_as_strided():
    buf = fill_bytes(4096, 1)
    for (c, b, s) in [(5, 3, 40), (4, 7, 7), (3, 2, 100)]:
        t = oracle.OType.basic("INT16").hvector(c, b, s)
        v = np.lib.stride_tricks.as_strided(buf, shape=(c, b * 2), strides=(s, 1))
        assert np.array_equal(oracle.pack(t, 1, buf), v.reshape(-1))


def test_block_cyclic_mask():
    """C3 (reading A18): element (r,c) selected iff (floor(r/nb)%2, floor(c/nb)%2)==(0,1);
    packed order column-major over the selected elements."""
    for n, nb in [(8, 2), (16, 2), (32, 4)]:
        rec, org, nbytes = c3_block_cyclic(n, nb)
        buf = fill_bytes(nbytes, 2)
        A = buf.view(np.float64).reshape(n, n).T
        r = np.arange(n)[:, None]
        c = np.arange(n)[None, :]
        mask = ((r // nb) % 2 == 0) & ((c // nb) % 2 == 1)
        exp = A.T[mask.T].view(np.uint8)      # column-major order of selected
        got = oracle.pack(oracle.from_recipe(rec), 1, buf, org)
        assert np.array_equal(got, exp)
        if n == 8:
            assert len(got) == 16 * 8


# ---------------------------------------------------------------- address encoding
def test_address_encoding_particles():
    """Source words hold their own byte offsets, so the packed stream IS the list of
    source addresses: compare with the hand-written particle typemap (A19)."""
    rec, _, nbytes = c5_particles(56 * 10, seed=1234)
    idx = rec[2] // 64
    buf = address_words(nbytes)
    got = oracle.pack(oracle.from_recipe(rec), 1, buf).view(np.uint32)
    per = [0] + [8 + 4 * k for k in range(12)] + [56]        # 4-byte words of one particle
    exp = np.concatenate([i * 64 + np.array(per) for i in idx]).astype(np.uint32)
    assert np.array_equal(got, exp)


# ---------------------------------------------------------------- twin vs oracle, brute force
def _tiny_types():
    I = ("basic", "INT32")
    Dd = ("basic", "DOUBLE")
    Bt = ("basic", "BYTE")
    out = []
    for c, b, s in itertools.product(range(0, 4), range(0, 4), range(-3, 4)):
        out.append(("vector", c, b, s, I))
    for bl in itertools.product(range(0, 3), repeat=3):
        for dp in [(0, 3, 6), (6, 0, 3), (1, 1, 5), (4, 2, 0)]:
            out.append(("indexed", list(bl), list(dp), I))
            out.append(("hindexed", list(bl), list(dp), Bt))
    for d0, d1 in itertools.product(range(0, 17, 3), range(0, 17, 4)):
        out.append(("struct", [1, 2], [d0, d1], [I, Dd]))
        out.append(("struct", [2, 1], [d0, d1], [("resized", I, -2, 8), Bt]))
    # derived old types whose extent != size (MPI-3.1 §4.1.2: strides and element
    # displacements count in extent(old) units) and structs whose largest basic
    # alignment is < 8 (the ε rule rounds to that alignment, reading A8)
    S16 = ("basic", "INT16")
    R8 = ("resized", I, 0, 8)
    SDI = ("struct", [1, 1], [0, 8], [Dd, I])
    SHB = ("struct", [1, 1], [0, 2], [S16, Bt])
    for old in (R8, SDI, SHB, ("resized", Bt, -1, 3)):
        for c, b, s in itertools.product(range(1, 4), range(1, 3), (-2, 1, 3)):
            out.append(("vector", c, b, s, old))
        for dp in [(0, 2), (3, 0), (1, 5)]:
            out.append(("indexed", [1, 2], list(dp), old))
            out.append(("indexed_block", 2, list(dp), old))
            out.append(("hindexed", [2, 1], [dp[0] * 5, dp[1] * 7], old))
    for d0, d1 in itertools.product(range(0, 9, 2), range(0, 9, 3)):
        out.append(("struct", [1, 1], [d0, d1], [S16, Bt]))
        out.append(("struct", [2, 1], [d0, d1], [Bt, ("basic", "FLOAT")]))
    out.append(("contiguous", 3, ("resized", ("vector", 3, 1, 3, Dd), 0, 8)))
    out.append(("contiguous", 3, ("vector", 2, 1, 3, Dd)))
    out.append(("hvector", 2, 2, 64, ("struct", [1, 1], [0, 8], [Dd, I])))
    out.append(("subarray", [3, 4, 2], [2, 2, 1], [1, 0, 1], "F", ("vector", 2, 1, 2, I)))
    out.append(("indexed_block", 2, [5, 0, 9], ("contiguous", 2, Bt)))
    out.append(("hindexed_block", 1, [64, 0, 128], PARTICLE))
    out.append(("resized", ("vector", 3, 1, 2, I), -4, 12))
    out.append(("contiguous", 2, ("resized", ("vector", 3, 1, 2, I), -4, 12)))
    return out


def test_twin_matches_oracle_enumerated():
    tys = _tiny_types()
    assert len(tys) > 300
    for r in tys:
        t = oracle.from_recipe(r)
        tw = ref.from_recipe(r)
        i = t.info()
        for k in ("size", "lb", "ub", "extent", "true_lb", "true_ub"):
            assert i[k] == getattr(tw, k), (r, k, i[k], getattr(tw, k))
        kk, dd = t.typemap()
        assert [(int(a), int(b)) for a, b in zip(kk, dd)] == tw.entries, r
        # pack of 2 instances over a buffer that covers every address
        span_lo = min(0, i["true_lb"], i["true_lb"] + i["extent"])
        span_hi = max(i["true_ub"], i["true_ub"] + i["extent"], 1)
        org = -span_lo + 8
        buf = fill_bytes(org + span_hi + 8, 99)
        a = oracle.pack(t, 2, buf, org)
        b = ref.pack(tw, 2, buf.tobytes(), org)
        assert a.tobytes() == b, r


def test_brute_force_pack_tiny():
    """Brute force: pack byte p equals buf[origin + k*extent + disp_j + (p - start_j)] where
    the typemap entry j of instance k covers stream byte p — enumerated independently of
    both the walk and the twin, from the typemap listing alone."""
    for r in _tiny_types()[::7]:
        t = oracle.from_recipe(r)
        i = t.info()
        kk, dd = t.typemap()
        sizes = np.array(oracle.BASIC_SIZE)[kk] if len(kk) else np.zeros(0, dtype=np.int64)
        org = 256
        buf = fill_bytes(1024, 5)
        exp = []
        for k in range(3):
            for kind, d, sz in zip(kk, dd, sizes):
                for b in range(sz):
                    exp.append(buf[org + k * i["extent"] + d + b])
        got = oracle.pack(t, 3, buf, org)
        assert got.tolist() == exp, r


# ---------------------------------------------------------------- unpack invariants, pos/len
@pytest.mark.parametrize("rname", ["tri", "sub", "face", "part"])
def test_unpack_roundtrip_and_gaps(rname):
    rec, org, nbytes = {
        "tri": c2_lower_triangle(37),
        "sub": c1_submatrix(9, 23, 2, 3),
        "face": c4_face("x+", 6, 1, True),
        "part": c5_particles(56 * 40),
    }[rname]
    t = oracle.from_recipe(rec)
    src = fill_bytes(nbytes, 21)
    packed = oracle.pack(t, 1, src, org)
    dst = poison(nbytes)
    oracle.unpack(t, 1, packed, dst, org)
    # covered bytes restored, every other byte still poison
    kk, dd = t.typemap()
    covered = np.zeros(nbytes, dtype=bool)
    for kind, d in zip(kk, dd):
        covered[org + d: org + d + oracle.BASIC_SIZE[kind]] = True
    assert np.array_equal(dst[covered], src[covered])
    assert np.all(dst[~covered] == 0xA5)
    # pack(unpack(y)) == y for a non-overlapping type
    y = fill_bytes(len(packed), 77)
    d2 = poison(nbytes)
    oracle.unpack(t, 1, y, d2, org)
    assert np.array_equal(oracle.pack(t, 1, d2, org), y)


def test_pos_len_concatenation():
    rec, org, nbytes = c1_submatrix(9, 23, 2, 3)
    t = oracle.from_recipe(rec)
    buf = fill_bytes(nbytes * 3, 4)
    whole = oracle.pack(t, 2, buf, org)
    rng = np.random.default_rng(0)
    for _ in range(20):
        cuts = np.sort(rng.integers(0, len(whole) + 1, size=5))
        cuts = [0] + list(cuts) + [len(whole)]
        parts = [oracle.pack(t, 2, buf, org, int(a), int(b - a)) for a, b in zip(cuts[:-1], cuts[1:])]
        assert np.array_equal(np.concatenate(parts), whole)
        # fragments unpacked in any order give the whole unpack
        d1 = poison(len(buf))
        oracle.unpack(t, 2, whole, d1, org)
        d2 = poison(len(buf))
        order = rng.permutation(len(parts))
        for j in order:
            oracle.unpack(t, 2, parts[j], d2, org, pos=int(cuts[j]))
        assert np.array_equal(d1, d2)
    assert len(oracle.pack(t, 2, buf, org, len(whole) + 5, 10)) == 0


@pytest.mark.parametrize("extent", [8, 16, 40, 2])
def test_pos_resume_overlapping_instances(extent):
    """Resuming at a stream position with count > 1 must seek instances by SIZE: instance
    k covers stream bytes [k*size, (k+1)*size) and sits at k*extent in memory (MPI-3.1
    §4.1.6; the fragment restart of [L18:c1430 §3.2]).  Closed form for a contiguous
    element resized to extent e (e < size: overlapping instances, legal to pack):
    stream byte p comes from address (p // size)*e + p % size."""
    size = 16
    rec = ("resized", ("contiguous", 4, ("basic", "INT32")), 0, extent)
    t = oracle.from_recipe(rec)
    count = 5
    n = count * size
    buf = fill_bytes(n * 4, 21)
    p = np.arange(n)
    whole = buf[(p // size) * extent + p % size]
    assert np.array_equal(oracle.pack(t, count, buf), whole)
    for pos in (1, 15, 16, 20, 33, 47, 64, 79):
        for ln in (1, 7, 16, 30, n):
            assert np.array_equal(oracle.pack(t, count, buf, 0, pos, ln), whole[pos:pos + ln]), (pos, ln)


def test_multithreaded_equals_single():
    rec, _, nbytes = c2_lower_triangle(300)
    t = oracle.from_recipe(rec)
    buf = fill_bytes(nbytes, 8)
    a = oracle.pack(t, 1, buf)
    b = oracle.pack(t, 1, buf, threads=7)
    assert np.array_equal(a, b)
    d1, d2 = poison(nbytes), poison(nbytes)
    oracle.unpack(t, 1, a, d1)
    oracle.unpack(t, 1, a, d2, threads=5)
    assert np.array_equal(d1, d2)


def test_addr_of_matches_typemap():
    rec, _, _ = c5_particles(56 * 20)
    t = oracle.from_recipe(rec)
    kk, dd = t.typemap()
    addrs = np.concatenate([np.arange(oracle.BASIC_SIZE[k]) + d for k, d in zip(kk, dd)])
    ps = np.array(sorted({0, 3, 4, 5, 55, 56, 57, 100, len(addrs) - 1}))
    assert np.array_equal(oracle.addr_of(t, 1, ps), addrs[ps])
    # count > 1: instance k shifted by k*extent
    ext = t.extent
    ps2 = ps + len(addrs)
    assert np.array_equal(oracle.addr_of(t, 2, ps2), addrs[ps] + ext)


def test_oracle_mutants_killed():
    """Each deliberate bug in oracle.c (tools/oracle_mutants.py: extent-vs-size scaling
    in the constructors' bounds and in the typemap walk, a dropped j*extent term, the
    struct ε rule, subarray order and starts, instance placement, fragment resume,
    pos handling of pack/unpack, resized/marker/true bounds) makes at least one pin above
    fail, and the unmutated oracle passes them in the tool's scratch copy."""
    import subprocess
    import sys
    tool = os.path.join(os.path.dirname(HERE), "tools", "oracle_mutants.py")
    r = subprocess.run([sys.executable, tool], capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout + r.stderr
