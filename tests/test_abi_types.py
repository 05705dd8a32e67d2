"""CPU tests of the C-ABI library (no GPU): it loads, exports every symbol
include/dt.h declares, and its host type system (constructors, bounds,
flattening into levels + block template, kernel plan, error codes) agrees with
the oracle.  T1 in SURVEY §4: expanding the library's normalised descriptor on
the host must give exactly the oracle's typemap (same byte addresses in the
same order)."""
import os
import re

import numpy as np
import pytest

import oracle
from paper_conf_hpdc_wubvjd16_b200 import dt
from workloads import (c1_submatrix, c2_lower_triangle, c3_block_cyclic, c4_face, c5_particles, c5b_irregular,
                       stair_triangle, upper_triangle)

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_library_exports_every_declared_symbol():
    hdr = open(os.path.join(ROOT, "include", "dt.h")).read()
    hdr = re.sub(r"/\*.*?\*/", "", hdr, flags=re.S)
    names = set(re.findall(r"\b(dt_[a-z0-9_]+)\s*\(", hdr))
    assert len(names) >= 30
    L = dt.lib()
    missing = [n for n in sorted(names) if not hasattr(L, n)]
    assert not missing, missing
    assert dt.lib().dt_version().decode().startswith("dt ")


def _oracle_blocks(ot, count):
    """Merged (disp, len) blocks of the oracle's typemap, count instances."""
    k, d = ot.typemap()
    ext = ot.extent
    sizes = np.array(oracle.BASIC_SIZE, dtype=np.int64)[k] if len(k) else np.zeros(0, np.int64)
    D, Ls = [], []
    for c in range(count):
        for disp, sz in zip(d + c * ext, sizes):
            if D and D[-1] + Ls[-1] == disp:
                Ls[-1] += int(sz)
            else:
                D.append(int(disp))
                Ls.append(int(sz))
    return np.array(D, dtype=np.int64), np.array(Ls, dtype=np.int64)


def _recipes():
    from tests.test_oracle_pins import _tiny_types
    out = list(_tiny_types())
    out += [c1_submatrix(9, 23, 2, 3)[0], c2_lower_triangle(40)[0], upper_triangle(17)[0], stair_triangle(24, 8)[0],
            c3_block_cyclic(32, 4)[0], c4_face("x-", 6)[0], c4_face("y+", 6, 1, True)[0], c4_face("z-", 6)[0],
            c5_particles(56 * 30)[0], c5b_irregular(700)[0]]
    return out


def test_bounds_match_oracle():
    for r in _recipes():
        o = oracle.from_recipe(r).info()
        t = dt.from_recipe(r)
        assert t.size == o["size"], r
        assert (t.lb, t.extent) == (o["lb"], o["extent"]), r
        assert t.true_extent == (o["true_lb"], o["true_ub"] - o["true_lb"]), r


@pytest.mark.parametrize("count", [1, 3])
def test_flatten_matches_oracle_typemap(count):
    for r in _recipes():
        ot = oracle.from_recipe(r)
        d0, l0 = _oracle_blocks(ot, count)
        d1, l1 = dt.from_recipe(r).flatten(count)
        assert np.array_equal(d0, d1) and np.array_equal(l0, l1), r


def test_forms_of_paper_workloads():
    # C1: V is one 2 KiB run repeated by one regular level (vector kernel, [L16:c2243 §3.1])
    f = dt.from_recipe(c1_submatrix()[0]).form()
    assert (f.nblocks, f.tsize, f.nlevels) == (1, 2048, 1)
    assert (f.level_count[0], f.level_stride[0]) == (256, 8192)
    # C2: T is a 4096-entry block list (DEV list, [L16:c5201 §3.2]), len_j=(4096-j)*8
    f = dt.from_recipe(c2_lower_triangle()[0]).form()
    assert (f.nblocks, f.nlevels, f.tsize) == (4096, 0, 67125248)
    # C3: 512 B runs; the column level merges with the row-block level (64 x 1 KiB = one column)
    f = dt.from_recipe(c3_block_cyclic()[0]).form()
    assert (f.nblocks, f.tsize, f.nlevels) == (1, 512, 2) and f.size == 1 << 27
    # C4 x-face: 4-byte elements under two regular levels; y/z faces: 2 KiB runs
    f = dt.from_recipe(c4_face("x-")[0]).form()
    assert (f.nblocks, f.tsize, f.nlevels) == (1, 4, 2)
    f = dt.from_recipe(c4_face("z+")[0]).form()
    assert (f.nblocks, f.tsize, f.nlevels) == (1, 2048, 1)
    # C5: particle template (0,4),(8,52) under one list level (the index list)
    rec = c5_particles(56 * 1000)[0]
    f = dt.from_recipe(rec).form()
    assert (f.nblocks, f.tsize, f.nlevels) == (2, 56, 1) and f.level_is_list[0] == 1
    d, ln = dt.from_recipe(rec[3]).flatten(1)
    assert list(d) == [0, 8] and list(ln) == [4, 52]


def test_plan_selects_kernels():
    t = dt.from_recipe(c2_lower_triangle()[0])
    assert t.plan(1, 0x10000, 0x20000, 0, 1 << 30) == (1, 8)     # long runs: warp segments
    t = dt.from_recipe(c4_face("x-")[0])
    assert t.plan(1, 0x10000, 0x20000, 0, 1 << 30)[0] == 4       # 4-byte elements: smem-staged gathers
    assert t.plan(1, 0x10000, 0x20004, 0, 1 << 30)[0] == 2       # packed side not 16-B aligned: word kernel
    k, g = t.plan(1, 0x10000, 0x20000, 0, 1 << 30)
    assert g == 4
    t = dt.from_recipe(c5_particles(56 * 100)[0])
    assert t.plan(1, 0x10000, 0x20000, 0, 1 << 30) == (6, 4)     # dense records: record spans
    assert t.plan(1, 0x10000, 0x20004, 0, 1 << 30) == (2, 4)     # packed side not 16-B aligned: words
    assert t.plan(1, 0x10008, 0x20000, 0, 1 << 30) == (4, 4)     # record bases not 16-B aligned: staged words
    assert t.plan(1, 0x10000, 0x20000, 32, 4000) == (6, 4)       # 16-B-congruent fragment
    # sparse records (8 of 32 span bytes) stay on word gathers (smem-staged)
    t = dt.from_recipe(("hvector", 100, 1, 64, ("resized", ("struct", [1, 1], [0, 28], [("basic", "INT32")] * 2),
                                                0, 64)))
    assert t.plan(1, 0x10000, 0x20000, 0, 800)[0] == 4
    # byte-granular start position lowers the word size
    assert t.plan(1, 0x10000, 0x20000, 3, 100) == (2, 1)
    # irregular short blocks under a template too large for a word table: block spans
    t = dt.from_recipe(c5b_irregular(1 << 20)[0])
    assert t.plan(1, 0x10000, 0x20000, 0, 1 << 20) == (7, 4)
    assert t.plan(1, 0x10000, 0x20008, 0, 1 << 20) == (7, 4)   # packed side only word-aligned
    assert t.plan(1, 0x10000, 0x20000, 1, 1 << 19) == (3, 1)   # byte words: block windows
    # ... unless the list is not locally dense (shuffled blocks / unsorted records): windows
    rec, _, _ = c5b_irregular(1 << 20)
    perm = np.random.default_rng(9).permutation(len(rec[1]))
    t = dt.from_recipe(("hindexed", rec[1][perm], rec[2][perm], rec[3]))
    assert t.plan(1, 0x10000, 0x20000, 0, 1 << 20) == (3, 4)
    rs = ("resized", ("struct", [1, 1], [0, 8], [("basic", "INT32"), ("basic", "DOUBLE")]), 0, 16)
    slots = np.random.default_rng(5).permutation(1 << 16)[: 1 << 15].astype(np.int64)
    t = dt.from_recipe(("hindexed", np.ones(1 << 15, dtype=np.int64), slots * 16, rs))
    assert t.plan(1, 0x10000, 0x20000, 0, 1 << 16)[0] == 6    # whole-record loads, any order
    assert t.plan(1, 0x10008, 0x20000, 0, 1 << 16)[0] == 4    # records not 16-B aligned: staged word table
    # contiguous type, many instances: one long run
    t = dt.Type.basic("DOUBLE").contiguous(10)
    assert t.plan(1000, 0x10000, 0x20000, 0, 80000)[0] == 1
    assert t.plan(1, 0, 0, 80, 10)[0] == 0                       # past the end: nothing


def test_error_codes():
    b = dt.Type.basic("INT32")
    with pytest.raises(dt.DTError) as e:
        b.vector(-1, 1, 1)
    assert e.value.name == "DT_ERR_ARG"
    with pytest.raises(dt.DTError) as e:
        b.subarray([4, 4], [2, 5], [0, 0])
    assert e.value.name == "DT_ERR_ARG"
    t = b.vector(4, 1, 2)                                         # never committed
    with pytest.raises(dt.DTError) as e:
        dt.pack(t, 1, 0x1000, 0x2000, stream=0)
    assert e.value.name == "DT_ERR_NOT_COMMITTED"
    assert dt.lib().dt_basic_type(42) is None


def test_component_free_is_safe():
    b = dt.Type.basic("DOUBLE")
    v = b.vector(3, 2, 5)
    c = v.contiguous(2)
    del v                                                         # drop our ref to the component
    import gc
    gc.collect()
    d, ln = c.flatten(1)
    assert c.size == 96 and d.tolist() == [0, 40, 80, 136, 176] and ln.tolist() == [16, 16, 32, 16, 16]


def test_type_serialize_roundtrip():
    """dt_type_serialize / dt_type_deserialize (shipping a receive layout to the sender
    of a direct plan): same bounds, same flattened typemap at several counts, usable
    as a component, malformed blobs rejected."""
    import numpy as np
    from workloads import c1_submatrix, c3_block_cyclic, c4_face
    recs = [c2_lower_triangle(300)[0], c3_block_cyclic(1024, 64)[0], c5_particles(56 * 100)[0], c4_face("x-", 40)[0],
            c1_submatrix(64, 200, 1, 2)[0], c5b_irregular(1 << 12)[0],
            ("resized", ("struct", [1, 1], [0, 16], [("basic", "DOUBLE")] * 2), -8, 40),
            ("vector", 3, 1, -2, ("basic", "INT32"))]
    for r in recs:
        t = dt.from_recipe(r)
        u = dt.Type.deserialize(t.serialize())
        assert (u.size, u.extent, u.true_extent) == (t.size, t.extent, t.true_extent)
        for count in (1, 3):
            d1, l1 = t.flatten(count)
            d2, l2 = u.flatten(count)
            assert np.array_equal(d1, d2) and np.array_equal(l1, l2)
        v = u.contiguous(2)
        assert v.size == 2 * t.size
    blob = bytearray(dt.from_recipe(recs[0]).serialize())
    for bad in (bytes(blob[:40]), bytes(blob[:-8]), b"\0" * len(blob)):
        with pytest.raises(dt.DTError) as e:
            dt.Type.deserialize(bad)
        assert e.value.name == "DT_ERR_ARG"


@pytest.mark.parametrize("threads", ["1", "7"])
def test_parallel_flatten_matches_numpy(threads, monkeypatch):
    """f2: type construction of a huge block list runs its bounds pass and copies on
    several host threads; the bounds and the flattened (merged) blocks must equal
    numpy's, for any thread count."""
    monkeypatch.setenv("DT_HOST_THREADS", threads)
    rng = np.random.default_rng(5)
    n = 3_000_000
    lens = rng.integers(1, 5, size=n) * 4
    gaps = rng.integers(0, 3, size=n) * 4  # a third of the gaps are 0: merges, also across ranges
    d = np.concatenate([[0], np.cumsum(lens + gaps)[:-1]])
    t = dt.Type.basic("BYTE").hindexed(lens, d)
    bd, bl = t.flatten(1)
    end = d + lens
    m = np.ones(n, bool)
    m[1:] = d[1:] != end[:-1]
    starts = np.flatnonzero(m)
    assert np.array_equal(bd, d[starts]) and np.array_equal(bl, np.add.reduceat(lens, starts))
    assert t.size == int(lens.sum()) and t.true_extent == (0, int(d[-1] + lens[-1]))
