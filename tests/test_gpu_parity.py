"""GPU parity (T2): libdt's CUDA pack/unpack vs the CPU oracle, byte for byte.

Bit-exact is the bar (pure byte movement; sources are splitmix64 words, so NaN
payloads and signed zeros must survive).  Destinations are poisoned 0xA5 with
4 KiB guard zones on both sides; unpack must leave every byte outside the
typemap untouched.  Workloads: SURVEY §8(d) configs C1-C5 (paper: V [L22:c1966],
T [L22:c2839], SHOC-style faces [L14:c1929], LAMMPS-style index lists
[L14:c2154]) at full size, plus random tiny types with ragged pos/len splits
and misaligned origins (prologue/epilogue [L16:c3618 §3.1]).
"""
import numpy as np
import pytest

import oracle
from workloads import (c1_submatrix, c2_lower_triangle, c3_block_cyclic, c4_face, c5_particles, c5b_irregular,
                       fill_bytes, stair_triangle, upper_triangle)

pytestmark = pytest.mark.gpu

GUARD = 4096


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    torch.cuda.init()
    return torch


def _dev(torch, host: np.ndarray):
    return torch.from_numpy(np.ascontiguousarray(host)).cuda()


def _poisoned(torch, n):
    return torch.full((n + 2 * GUARD,), 0xA5, dtype=torch.uint8, device="cuda")


def check_pack_unpack(torch, recipe, origin, parent, count=1, pos=0, nbytes=None, seed=1, origin_pad=0):
    from paper_conf_hpdc_wubvjd16_b200 import dt
    ot = oracle.from_recipe(recipe)
    t = dt.from_recipe(recipe).commit()
    ext = ot.extent
    span = parent + max(0, (count - 1) * ext)
    org = origin + origin_pad
    src_h = fill_bytes(span + origin_pad + 64, seed)
    total = count * ot.size
    n = max(0, min(total - pos, total if nbytes is None else nbytes))
    exp = oracle.pack(ot, count, src_h, org, pos, n)
    src_d = _dev(torch, src_h)
    out = _poisoned(torch, n)
    got_n = dt.pack(t, count, src_d, out.data_ptr() + GUARD, pos, n, origin_offset=org)
    torch.cuda.synchronize()
    assert got_n == n
    o = out.cpu().numpy()
    assert np.all(o[:GUARD] == 0xA5) and np.all(o[GUARD + n:] == 0xA5), "pack wrote outside its output"
    assert np.array_equal(o[GUARD:GUARD + n], exp), "pack mismatch"
    # unpack the oracle's bytes into a poisoned layout
    dst_h = np.full(span + origin_pad + 64, 0xA5, dtype=np.uint8)
    oracle.unpack(ot, count, exp, dst_h, org, pos)
    dst_d = _poisoned(torch, len(dst_h))
    pk = _dev(torch, exp) if n else torch.zeros(1, dtype=torch.uint8, device="cuda")
    got_n = dt.unpack(t, count, pk, dst_d.data_ptr() + GUARD, pos, n, origin_offset=org)
    torch.cuda.synchronize()
    assert got_n == n
    d = dst_d.cpu().numpy()
    assert np.all(d[:GUARD] == 0xA5) and np.all(d[GUARD + len(dst_h):] == 0xA5), "unpack wrote outside the span"
    assert np.array_equal(d[GUARD:GUARD + len(dst_h)], dst_h), "unpack mismatch"


def _oracle_overlaps(ot, count):
    """True iff the typemap of `count` instances has two entries sharing a byte
    (reading A9: such a map may be packed but not unpacked)."""
    kk, dd = ot.typemap()
    ext = ot.extent
    iv = sorted((k * ext + int(d), k * ext + int(d) + oracle.BASIC_SIZE[int(kind)])
                for k in range(count) for kind, d in zip(kk, dd))
    return any(b[0] < a[1] for a, b in zip(iv, iv[1:]))


def check_or_overlap(torch, r, origin, parent, count, **kw):
    """check_pack_unpack; a DT_ERR_OVERLAP is accepted only when the oracle's own
    typemap of `count` instances really overlaps (no silent false rejection)."""
    try:
        check_pack_unpack(torch, r, origin, parent, count=count, **kw)
    except Exception as e:  # noqa: BLE001
        if "DT_ERR_OVERLAP" not in str(e):
            raise
        assert _oracle_overlaps(oracle.from_recipe(r), count), ("false DT_ERR_OVERLAP", r, count)


def check_empty(torch, recipe, count, pos=0, nbytes=64):
    """Count 0 or size 0 (SURVEY §8(b) errors): DT_OK, 0 bytes, nothing written."""
    from paper_conf_hpdc_wubvjd16_b200 import dt
    t = dt.from_recipe(recipe).commit()
    src = torch.full((4096,), 0x5A, dtype=torch.uint8, device="cuda")
    out = _poisoned(torch, 64)
    assert dt.pack(t, count, src.data_ptr() + 2048, out.data_ptr() + GUARD, pos, nbytes) == 0
    dst = _poisoned(torch, 4096)
    pk = torch.full((64,), 0x3C, dtype=torch.uint8, device="cuda")
    assert dt.unpack(t, count, pk, dst.data_ptr() + GUARD + 2048, pos, nbytes) == 0
    torch.cuda.synchronize()
    assert bool((out == 0xA5).all()) and bool((dst == 0xA5).all()), "empty request wrote bytes"


# ------------------------------------------------------------------ the paper's workloads at full size
@pytest.mark.parametrize("r0c0", [(0, 0), (1, 1), (3, 7)])
def test_c1_submatrix(torch_cuda, r0c0):
    rec, org, parent = c1_submatrix(256, 1024, *r0c0)
    check_pack_unpack(torch_cuda, rec, org, parent)


def test_c2_lower_triangle_full(torch_cuda):
    rec, org, parent = c2_lower_triangle(4096)
    check_pack_unpack(torch_cuda, rec, org, parent, seed=0x5EED0002)


@pytest.mark.parametrize("n", [1, 2, 33, 1000])
def test_triangles_small(torch_cuda, n):
    for mk in (c2_lower_triangle, upper_triangle):
        rec, org, parent = mk(n)
        check_pack_unpack(torch_cuda, rec, org, parent)
    rec, org, parent = stair_triangle(max(n, 64), 32)
    check_pack_unpack(torch_cuda, rec, org, parent)


def test_c3_block_cyclic_full(torch_cuda):
    rec, org, parent = c3_block_cyclic(8192, 64)
    check_pack_unpack(torch_cuda, rec, org, parent, seed=0x5EED0003)


@pytest.mark.parametrize("face", ["x-", "x+", "y-", "y+", "z-", "z+"])
@pytest.mark.parametrize("ghost", [False, True])
def test_c4_halo_faces_full(torch_cuda, face, ghost):
    rec, org, parent = c4_face(face, 512, 1, ghost)
    check_pack_unpack(torch_cuda, rec, org, parent, seed=0x5EED0004)


@pytest.mark.parametrize("m", [1 << 10, 1 << 16, 1 << 22, 1 << 26])
def test_c5_particles(torch_cuda, m):
    rec, org, parent = c5_particles(m)
    check_pack_unpack(torch_cuda, rec, org, parent, seed=0x5EED0005)


@pytest.mark.parametrize("m", [1 << 10, 1 << 20])
def test_c5b_irregular(torch_cuda, m):
    rec, org, parent = c5b_irregular(m)
    check_pack_unpack(torch_cuda, rec, org, parent, seed=0x5EED0006)


# ------------------------------------------------------------------ resume from a byte position
@pytest.mark.parametrize("name", ["C1", "C2", "C4x", "C5"])
def test_pos_len_fragments(torch_cuda, name):
    mk = {"C1": lambda: c1_submatrix(64, 200, 1, 2), "C2": lambda: c2_lower_triangle(300),
          "C4x": lambda: c4_face("x+", 40), "C5": lambda: c5_particles(56 * 500)}[name]
    rec, org, parent = mk()
    rng = np.random.default_rng(7)
    size = oracle.from_recipe(rec).size
    for count in (1, 2):
        total = size * count
        for _ in range(4):
            a, b = sorted(rng.integers(0, total + 1, size=2))
            check_pack_unpack(torch_cuda, rec, org, parent, count=count, pos=int(a), nbytes=int(b - a))


def test_concatenated_fragments_equal_whole(torch_cuda):
    import torch
    from paper_conf_hpdc_wubvjd16_b200 import dt
    rec, org, parent = c2_lower_triangle(512)
    t = dt.from_recipe(rec).commit()
    src = _dev(torch, fill_bytes(parent, 3))
    n = t.size
    whole = torch.empty(n, dtype=torch.uint8, device="cuda")
    dt.pack(t, 1, src, whole)
    cuts = [0, 1, 7, 4096, 4097, 100000, n - 3, n]
    parts = torch.empty(n, dtype=torch.uint8, device="cuda")
    for a, b in zip(cuts[:-1], cuts[1:]):
        dt.pack(t, 1, src, parts.data_ptr() + a, a, b - a)
    torch.cuda.synchronize()
    assert torch.equal(whole, parts)


# ------------------------------------------------------------------ random tiny types, misaligned origins
def test_random_tiny_types(torch_cuda):
    from tests.test_oracle_pins import _tiny_types
    rng = np.random.default_rng(11)
    tys = _tiny_types()
    for i, r in enumerate(tys[::3]):
        ot = oracle.from_recipe(r)
        info = ot.info()
        if info["size"] == 0:   # size 0: DT_OK, no bytes, nothing written
            check_empty(torch_cuda, r, int(rng.integers(0, 4)))
            continue
        lo = min(0, info["true_lb"], info["true_lb"] + 2 * info["extent"])
        hi = max(info["true_ub"], info["true_ub"] + 2 * info["extent"], 1)
        count = int(rng.integers(1, 4))
        total = count * info["size"]
        a, b = sorted(rng.integers(0, total + 1, size=2))
        # overlapping typemaps are only packed (unpack is rejected, reading A9)
        check_or_overlap(torch_cuda, r, -lo + 16, hi - lo + 32, count, pos=int(a), nbytes=int(b - a),
                         seed=i, origin_pad=int(rng.integers(0, 16)))


@pytest.mark.parametrize("kind", ["1", "2", "3", "4", "6", "7"])
@pytest.mark.parametrize("name", ["C1b", "C2s", "C3s", "C4x", "C4y", "C5", "C5b", "ctg"])
def test_every_kernel_family(torch_cuda, kind, name, monkeypatch):
    """Every kernel family (1 warp segments, 2 word table, 3 block windows, 4 smem/TMA
    staging, 6 record spans) on every workload it accepts, forced through DT_FORCE_KERNEL, with
    ragged pos/len (the planner falls back when a family does not apply)."""
    mk = {"C1b": lambda: c1_submatrix(256, 1024, 1, 1), "C2s": lambda: c2_lower_triangle(700),
          "C3s": lambda: c3_block_cyclic(1024, 64), "C4x": lambda: c4_face("x+", 96),
          "C4y": lambda: c4_face("y-", 96, 1, True), "C5": lambda: c5_particles(1 << 20),
          "C5b": lambda: c5b_irregular(1 << 20), "ctg": lambda: (("contiguous", 3000, ("basic", "INT32")), 0, 12000)}
    rec, org, parent = mk[name]()
    monkeypatch.setenv("DT_FORCE_KERNEL", kind)
    size = oracle.from_recipe(rec).size
    check_pack_unpack(torch_cuda, rec, org, parent)
    check_pack_unpack(torch_cuda, rec, org, parent, count=2, pos=48, nbytes=2 * size - 48 - 16)
    check_pack_unpack(torch_cuda, rec, org, parent, pos=20, nbytes=size - 37)


@pytest.mark.parametrize("extent", [8, 2, 40])
def test_resume_overlapping_instances(torch_cuda, extent):
    """count > 1 instances whose extent is smaller than their size (overlapping, pack-only)
    or larger: every kernel resumes at stream position p in instance p // size
    (the oracle pin test_pos_resume_overlapping_instances fixes the closed form)."""
    rec = ("resized", ("contiguous", 4, ("basic", "INT32")), 0, extent)
    for count in (3, 7):
        for pos, nbytes in ((0, None), (1, 30), (16, 16), (20, 100), (47, 5)):
            check_or_overlap(torch_cuda, rec, 16, 16 + count * 64 + 64, count, pos=pos, nbytes=nbytes)


@pytest.mark.parametrize("slice_", ["2048", "16384"])
def test_warp_segments_multi_wave(torch_cuda, slice_, monkeypatch):
    """The long-run kernel with fixed slices (several waves of short CTAs, as for streams of
    more than 128 KiB per warp of one wave): triangles, a block-cyclic vector and a skewed
    indexed list, whole streams, counts 2 and ragged fragments."""
    monkeypatch.setenv("DT_SEG_SLICE", slice_)
    for rec, org, parent in (c2_lower_triangle(700), stair_triangle(640, 64), c1_submatrix(300, 700, 3, 5)):
        size = oracle.from_recipe(rec).size
        check_pack_unpack(torch_cuda, rec, org, parent)
        check_pack_unpack(torch_cuda, rec, org, parent, count=2, pos=8, nbytes=2 * size - 24)
        check_pack_unpack(torch_cuda, rec, org, parent, pos=4096 + 8, nbytes=size // 3)


def test_full_size_sampled_long_vector(torch_cuda):
    """A 512 MiB column sub-matrix (V8K: 8192 columns of 64 KiB at a 128 KiB pitch) -- long
    enough for the multi-wave 16 KiB slices of the single-block kernel: 200k sampled stream
    bytes against the vector's closed form (stream byte p = column p // 64 KiB, byte
    p % 64 KiB), then unpack -> pack round trip."""
    import torch
    from paper_conf_hpdc_wubvjd16_b200 import dt
    rec, org, parent = c1_submatrix(8192, 16384)
    t = dt.from_recipe(rec).commit()
    n = t.size
    assert n == 8192 * 8192 * 8
    src = torch.empty(parent, dtype=torch.uint8, device="cuda").random_(0, 256)
    out = torch.empty(n, dtype=torch.uint8, device="cuda")
    dt.pack(t, 1, src, out, origin_offset=org)
    torch.cuda.synchronize()
    rng = np.random.default_rng(8)
    ps = np.unique(np.concatenate([rng.integers(0, n, size=200000), [0, n - 1]]))
    addr = (ps // 65536) * (16384 * 8) + ps % 65536 + org
    pt = torch.from_numpy(ps).cuda()
    assert torch.equal(out[pt], src[torch.from_numpy(addr).cuda()])
    dst = torch.zeros_like(src)
    dt.unpack(t, 1, out, dst, origin_offset=org)
    back = torch.empty_like(out)
    dt.pack(t, 1, dst, back, origin_offset=org)
    torch.cuda.synchronize()
    assert torch.equal(back, out)


@pytest.mark.parametrize("nbytes", [16, 4096, (1 << 20) + 16, 64 << 20])
def test_contiguous_run_copy(torch_cuda, nbytes):
    """A contiguous layout (one run after normalisation) moves with the grid-stride run
    copy when the run, the packed side and the length are 16-byte aligned, else with the
    warp-slice kernel: whole streams, 16-aligned and misaligned fragments, count > 1."""
    rec = ("contiguous", nbytes // 8, ("basic", "DOUBLE"))
    check_pack_unpack(torch_cuda, rec, 0, nbytes)
    check_pack_unpack(torch_cuda, rec, 16, nbytes, origin_pad=16)
    if nbytes >= 4096:
        check_pack_unpack(torch_cuda, rec, 0, nbytes, pos=32, nbytes=nbytes // 2)
        check_pack_unpack(torch_cuda, rec, 0, nbytes, pos=8, nbytes=nbytes // 2 + 8)
    check_pack_unpack(torch_cuda, rec, 0, nbytes, count=3)


def test_unpack_rejects_overlap(torch_cuda):
    import torch
    from paper_conf_hpdc_wubvjd16_b200 import dt
    t = dt.Type.basic("INT32").vector(4, 3, 2).commit()    # stride < blocklen: overlapping
    buf = torch.zeros(1024, dtype=torch.uint8, device="cuda")
    pk = torch.zeros(t.size, dtype=torch.uint8, device="cuda")
    dt.pack(t, 1, buf, pk)                                   # pack of an overlapping map is legal
    with pytest.raises(dt.DTError) as e:
        dt.unpack(t, 1, pk, buf)
    assert e.value.name == "DT_ERR_OVERLAP"


def test_host_pointer_rejected(torch_cuda):
    from paper_conf_hpdc_wubvjd16_b200 import dt
    t = dt.Type.basic("DOUBLE").vector(4, 1, 2).commit()
    h = np.zeros(256, dtype=np.uint8)
    import torch
    d = torch.zeros(256, dtype=torch.uint8, device="cuda")
    with pytest.raises(dt.DTError) as e:
        dt.pack(t, 1, h.ctypes.data, d)
    assert e.value.name == "DT_ERR_ARG"


def test_host_entry_points(torch_cuda):
    """dt_pack_host / dt_unpack_host (the e2e path): host buffers in and out."""
    from paper_conf_hpdc_wubvjd16_b200 import dt
    rec, org, parent = c2_lower_triangle(700)
    ot = oracle.from_recipe(rec)
    t = dt.from_recipe(rec).commit()
    src = fill_bytes(parent, 5)
    out = np.zeros(t.size, dtype=np.uint8)
    dt.pack_host(t, 1, src.ctypes.data + org, out.ctypes.data, stream=0)
    assert np.array_equal(out, oracle.pack(ot, 1, src, org))
    dst = np.full(parent, 0xA5, dtype=np.uint8)
    dt.unpack_host(t, 1, out.ctypes.data, dst.ctypes.data + org, stream=0)
    exp = np.full(parent, 0xA5, dtype=np.uint8)
    oracle.unpack(ot, 1, out, exp, org)
    assert np.array_equal(dst, exp)


@pytest.mark.parametrize("name", ["C2s", "C5", "C4x"])
def test_host_entry_points_pinned(torch_cuda, name):
    """Pinned host buffers: the kernels read/write host memory directly (zero-copy);
    bit-exact vs the oracle, fragments, and host gap bytes untouched by unpack."""
    import torch
    from paper_conf_hpdc_wubvjd16_b200 import dt
    rec, org, parent = {"C2s": lambda: c2_lower_triangle(700), "C5": lambda: c5_particles(56 * 5000),
                        "C4x": lambda: c4_face("x+", 48)}[name]()
    ot = oracle.from_recipe(rec)
    t = dt.from_recipe(rec).commit()
    src_h = fill_bytes(parent, 15)
    src = torch.from_numpy(src_h).pin_memory()
    n = t.size
    out = torch.full((n,), 0xA5, dtype=torch.uint8).pin_memory()
    dt.pack_host(t, 1, src.data_ptr() + org, out.data_ptr(), stream=0)
    exp = oracle.pack(ot, 1, src_h, org)
    assert np.array_equal(out.numpy(), exp)
    for a, b in ((0, n // 3), (n // 3, n - 5), (n - 5, n)):   # fragments at ragged positions
        part = torch.full((b - a,), 0xA5, dtype=torch.uint8).pin_memory()
        dt.pack_host(t, 1, src.data_ptr() + org, part.data_ptr(), a, b - a, stream=0)
        assert np.array_equal(part.numpy(), exp[a:b])
    dst = torch.full((parent,), 0xA5, dtype=torch.uint8).pin_memory()
    dt.unpack_host(t, 1, out.data_ptr(), dst.data_ptr() + org, stream=0)
    ref = np.full(parent, 0xA5, dtype=np.uint8)
    oracle.unpack(ot, 1, exp, ref, org)
    assert np.array_equal(dst.numpy(), ref)


@pytest.mark.parametrize("chunk", [None, str(1 << 20), str(3 << 20)])
@pytest.mark.parametrize("pipe", ["1", "2"])
@pytest.mark.parametrize("name", ["C2", "C5b"])
def test_host_pipeline_pinned(torch_cuda, name, chunk, pipe, monkeypatch):
    """Pinned host buffers above 8 MiB: the host-link pipeline (zero-copy gather/scatter on
    the SMs into a device chunk ring, copy engine for the packed side, two internal streams)
    is bit-exact vs the oracle for whole streams and a ragged fragment, at chunk sizes that
    do and do not divide the stream; unpack leaves the host gap bytes untouched."""
    import torch
    from paper_conf_hpdc_wubvjd16_b200 import dt
    if chunk:
        monkeypatch.setenv("DT_HOST_CHUNK", chunk)
    monkeypatch.setenv("DT_HOST_PIPE", pipe)  # 1: unpack pipelined, 2: pack too
    rec, org, parent = {"C2": lambda: c2_lower_triangle(), "C5b": lambda: c5b_irregular(24 << 20)}[name]()
    ot = oracle.from_recipe(rec)
    t = dt.from_recipe(rec).commit()
    src_h = fill_bytes(parent, 17)
    src = torch.from_numpy(src_h).pin_memory()
    n = t.size
    exp = oracle.pack(ot, 1, src_h, org)
    out = torch.full((n,), 0xA5, dtype=torch.uint8).pin_memory()
    dt.pack_host(t, 1, src.data_ptr() + org, out.data_ptr(), stream=0)
    assert np.array_equal(out.numpy(), exp)
    a, b = 4100, n - 9000  # fragment: ragged both ends
    part = torch.full((b - a,), 0xA5, dtype=torch.uint8).pin_memory()
    dt.pack_host(t, 1, src.data_ptr() + org, part.data_ptr(), a, b - a, stream=0)
    assert np.array_equal(part.numpy(), exp[a:b])
    dst = torch.full((parent,), 0xA5, dtype=torch.uint8).pin_memory()
    dt.unpack_host(t, 1, out.data_ptr(), dst.data_ptr() + org, stream=0)
    ref = np.full(parent, 0xA5, dtype=np.uint8)
    oracle.unpack(ot, 1, exp, ref, org)
    assert np.array_equal(dst.numpy(), ref)


def test_full_size_sampled_c5_large(torch_cuda):
    """BASELINE sizes where the oracle cannot produce the whole stream quickly:
    compare sampled stream bytes against the oracle's per-position addresses."""
    import torch
    from paper_conf_hpdc_wubvjd16_b200 import dt
    rec, org, parent = c5_particles(1 << 30)
    ot = oracle.from_recipe(rec)
    t = dt.from_recipe(rec).commit()
    src_h = fill_bytes(parent, 0x5EED0005)
    src = _dev(torch, src_h)
    n = t.size
    out = torch.empty(n, dtype=torch.uint8, device="cuda")
    dt.pack(t, 1, src, out)
    torch.cuda.synchronize()
    rng = np.random.default_rng(5)
    ps = np.unique(np.concatenate([rng.integers(0, n, size=200000), [0, n - 1]]))
    addr = oracle.addr_of(ot, 1, ps)
    got = out[torch.from_numpy(ps).cuda()].cpu().numpy()
    assert np.array_equal(got, src_h[org + addr])
    # unpack then re-pack equals the packed stream (untouched-gap check on a sample)
    dst = torch.full((parent,), 0xA5, dtype=torch.uint8, device="cuda")
    dt.unpack(t, 1, out, dst)
    back = torch.empty_like(out)
    dt.pack(t, 1, dst, back)
    torch.cuda.synchronize()
    assert torch.equal(back, out)
    covered = np.zeros(parent, dtype=bool)
    covered[org + addr] = True
    gaps = np.flatnonzero(~covered)[:: 97]
    idx = rec[2][:2000] + 4  # bytes 4..7 of a selected particle are padding: never written
    assert np.all(dst[torch.from_numpy(idx).cuda()].cpu().numpy() == 0xA5)
    del gaps


def test_full_size_sampled_c5b_1g_gpu_flatten(torch_cuda):
    """C5b at 1 GiB (3.0e7 irregular 4..64-byte blocks) committed through the GPU-side
    flattening (f2, the default for lists this long) and packed / unpacked by the
    block-span kernel: 200k sampled stream bytes against the oracle's per-position
    addresses, the unpack -> pack round trip, and sampled gap bytes left untouched."""
    import torch
    from paper_conf_hpdc_wubvjd16_b200 import dt
    rec, org, parent = c5b_irregular(1 << 30)
    ot = oracle.from_recipe(rec)
    t = dt.from_recipe(rec).commit()
    fi = t.form()
    assert fi.tsize == ot.size == 1 << 30
    src_h = fill_bytes(parent, 0x5EED0015)
    src = _dev(torch, src_h)
    n = t.size
    out = torch.empty(n, dtype=torch.uint8, device="cuda")
    dt.pack(t, 1, src, out)
    torch.cuda.synchronize()
    rng = np.random.default_rng(15)
    ps = np.unique(np.concatenate([rng.integers(0, n, size=200000), [0, n - 1]]))
    addr = oracle.addr_of(ot, 1, ps)
    got = out[torch.from_numpy(ps).cuda()].cpu().numpy()
    assert np.array_equal(got, src_h[org + addr])
    del src
    dst = torch.full((parent,), 0xA5, dtype=torch.uint8, device="cuda")
    dt.unpack(t, 1, out, dst)
    back = torch.empty_like(out)
    dt.pack(t, 1, dst, back)
    torch.cuda.synchronize()
    assert torch.equal(back, out)
    lens, disp = rec[1], rec[2]
    gap_at = disp[:-1] + lens[:-1]
    has_gap = np.flatnonzero(disp[1:] > gap_at)[:: 101][:20000]
    assert len(has_gap) > 1000
    assert np.all(dst[torch.from_numpy(gap_at[has_gap]).cuda()].cpu().numpy() == 0xA5)


# ------------------------------------------------------------------ record-span kernel (k_rec)
REC_TYPES = {
    # C5 particle records (G = 4): blocks (0,4),(8,52) of a 64-byte span
    "particle": lambda: c5_particles(56 * 3001),
    # struct{f64@0, f64@16} resized to 32 B, an array of them (G = 8, half payload)
    "pair8": lambda: (("contiguous", 1500, ("resized", ("struct", [1, 1], [0, 16], [("basic", "DOUBLE")] * 2),
                                           0, 32)), 0, 1500 * 32),
    # 16-byte runs at a 48-byte pitch, span 16 (G = 16)
    "run16": lambda: (("hvector", 2000, 1, 48, ("contiguous", 2, ("basic", "DOUBLE"))), 0, 2000 * 48),
    # two-level nest of 3-word records (span 16, 12 of 16 bytes), G = 4
    "nest4": lambda: (("hvector", 37, 1, 16 * 64 + 32, ("hvector", 64, 1, 16, ("contiguous", 3, ("basic", "INT32")))),
                      0, 37 * (16 * 64 + 32)),
}


@pytest.mark.parametrize("name", sorted(REC_TYPES))
def test_record_span_kernel(torch_cuda, name):
    """k_rec is the planner's choice for short blocks in small dense records and is
    bit-exact for whole streams, counts > 1 and ragged 16-aligned pos / G-granular len
    (records cut at both ends of a fragment)."""
    from paper_conf_hpdc_wubvjd16_b200 import dt
    rec, org, parent = REC_TYPES[name]()
    t = dt.from_recipe(rec).commit()
    assert t.plan(1, 4096, 8192, 0, t.size)[0] == 6
    size = t.size
    check_pack_unpack(torch_cuda, rec, org, parent, seed=31)
    rng = np.random.default_rng(3)
    for count in (1, 3):
        total = count * size
        for _ in range(3):
            a = int(rng.integers(0, total // 16)) * 16
            b = int(rng.integers(a // 4, total // 4 + 1)) * 4
            check_pack_unpack(torch_cuda, rec, org, parent, count=count, pos=a, nbytes=b - a, seed=a)


def _hindexed(lens, disp):
    return ("hindexed", np.asarray(lens, dtype=np.int64), np.asarray(disp, dtype=np.int64), ("basic", "BYTE"))


def _span_types():
    rng = np.random.default_rng(77)
    out = {}
    # C5b-like blocks, typemap order != address order (shuffled within groups of 48 blocks)
    n = 20000
    lens = rng.integers(1, 17, n) * 4
    gaps = rng.integers(0, 16, n) * 4
    disp = np.concatenate([[0], np.cumsum(lens[:-1] + gaps[:-1])])
    perm = np.concatenate([rng.permutation(48) + i for i in range(0, n - n % 48, 48)] + [np.arange(n - n % 48, n)])
    out["shuffled4"] = (_hindexed(lens[perm], disp[perm]), 0, int(disp[-1] + lens[-1]))
    # occasional 8 KiB jumps: windows alternate between the span path and the wide fallback
    gaps2 = gaps.copy()
    gaps2[::37] = 8192
    disp2 = np.concatenate([[0], np.cumsum(lens[:-1] + gaps2[:-1])])
    out["jumps4"] = (_hindexed(lens, disp2), 0, int(disp2[-1] + lens[-1]))
    # 8- and 16-byte granular blocks (G = 8, 16)
    for g in (8, 16):
        l8 = rng.integers(1, 9, n) * g
        g8 = rng.integers(0, 5, n) * g
        d8 = np.concatenate([[0], np.cumsum(l8[:-1] + g8[:-1])])
        out[f"gran{g}"] = (_hindexed(l8, d8), 0, int(d8[-1] + l8[-1]))
    # negative and descending displacements (origin inside the buffer)
    dd = -disp[:5000][::-1] - lens[:5000][::-1]
    span = int(disp[4999] + lens[4999])
    out["descending"] = (_hindexed(lens[:5000][::-1], dd), span, span + 64)
    # small irregular template repeated (count > 1): windows wrap across elements
    l3 = rng.integers(1, 9, 45) * 4
    d3 = np.concatenate([[0], np.cumsum(l3[:-1] + 12)])
    ext = int(d3[-1] + l3[-1] + 4)
    out["repeat"] = (("resized", _hindexed(l3, d3), 0, ext), 0, ext)
    return out


SPAN_TYPES = _span_types()


@pytest.mark.parametrize("name", sorted(SPAN_TYPES))
def test_block_span_kernel(torch_cuda, name, monkeypatch):
    """k_span (short blocks of a large irregular list): the planner's choice for C5b-like
    lists; bit-exact on unsorted, descending and jumping displacements, G = 4/8/16,
    element wrap-around inside a window (forced), and ragged pos/len."""
    from paper_conf_hpdc_wubvjd16_b200 import dt
    rec, org, parent = SPAN_TYPES[name]
    t = dt.from_recipe(rec).commit()
    if name == "repeat":
        monkeypatch.setenv("DT_FORCE_KERNEL", "7")
    else:
        assert t.plan(1, 4096, 8192, 0, t.size)[0] == 7
    size = t.size
    check_pack_unpack(torch_cuda, rec, org, parent, seed=5)
    rng = np.random.default_rng(11)
    for count in (1, 3):
        total = count * size
        for _ in range(3):
            a = int(rng.integers(0, total // 4)) * 4
            b = int(rng.integers(a // 4, total // 4 + 1)) * 4
            check_pack_unpack(torch_cuda, rec, org, parent, count=count, pos=a, nbytes=b - a, seed=a)


def test_random_types_forced_block_spans(torch_cuda, monkeypatch):
    """Tiny random types (the oracle pins' enumeration, another third of it) forced through
    the block-span kernel where it applies (G >= 4; the planner falls back otherwise), with
    counts 1-3, ragged pos/len and misaligned origins."""
    from tests.test_oracle_pins import _tiny_types
    monkeypatch.setenv("DT_FORCE_KERNEL", "7")
    rng = np.random.default_rng(12)
    for i, r in enumerate(_tiny_types()[1::3]):
        info = oracle.from_recipe(r).info()
        if info["size"] == 0:
            check_empty(torch_cuda, r, int(rng.integers(0, 4)))
            continue
        lo = min(0, info["true_lb"], info["true_lb"] + 2 * info["extent"])
        hi = max(info["true_ub"], info["true_ub"] + 2 * info["extent"], 1)
        count = int(rng.integers(1, 4))
        total = count * info["size"]
        a, b = sorted(rng.integers(0, total + 1, size=2))
        check_or_overlap(torch_cuda, r, -lo + 16, hi - lo + 32, count, pos=int(a), nbytes=int(b - a),
                         seed=i, origin_pad=int(rng.integers(0, 16)))


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_random_irregular_struct_lists(torch_cuda, seed):
    """Seeded random index lists of small structs (int32 + double pairs, resized records,
    random signed displacements, random block counts per entry) -- the nested
    struct/hindexed family of config C5 with irregular blocks -- through the planner's
    choice, whole streams and random 4-byte-aligned fragments, counts 1 and 2."""
    rng = np.random.default_rng(100 + seed)
    rec_sz = int(rng.choice([16, 24, 32]))
    rec = ("resized", ("struct", [1, 1], [0, 8], [("basic", "INT32"), ("basic", "DOUBLE")]), 0, rec_sz)
    n = int(rng.integers(3000, 9000))
    slots = rng.permutation(4 * n)[:n] - n  # signed, unsorted record slots
    bl = rng.integers(1, 4, size=n)
    rec_t = ("hindexed", bl, slots.astype(np.int64) * rec_sz * 4, rec)
    lo_slot, hi_slot = int(slots.min()), int(slots.max())
    org = -lo_slot * rec_sz * 4 + 64
    parent = (hi_slot - lo_slot) * rec_sz * 4 + 4 * rec_sz * 4 + 128
    size = oracle.from_recipe(rec_t).size
    ext = oracle.from_recipe(rec_t).extent
    check_pack_unpack(torch_cuda, rec_t, org, parent + ext, seed=seed)
    for count in (1, 2):
        total = count * size
        a = int(rng.integers(0, total // 4)) * 4
        b = int(rng.integers(a // 4, total // 4 + 1)) * 4
        check_pack_unpack(torch_cuda, rec_t, org, parent + ext, count=count, pos=a, nbytes=b - a, seed=a)


# ------------------------------------------------------------------ derived old types (VERDICT r01 pin gap)
_R8 = ("resized", ("basic", "INT32"), 0, 8)
_SDI = ("struct", [1, 1], [0, 8], [("basic", "DOUBLE"), ("basic", "INT32")])
_SHB = ("struct", [1, 1], [0, 2], [("basic", "INT16"), ("basic", "BYTE")])


def _transpose(n):
    """MPI transpose idiom: contiguous(N, resized(vector(N,1,N,DOUBLE),0,8)) reads an
    N x N column-major f64 matrix row by row (extent 8 per column type)."""
    return ("contiguous", n, ("resized", ("vector", n, 1, n, ("basic", "DOUBLE")), 0, 8)), 0, n * n * 8


@pytest.mark.parametrize("name", ["vec_resized", "idx_struct", "iblk_resized", "vec_struct16", "hidx_struct",
                                  "transpose64", "transpose300"])
def test_derived_old_types(torch_cuda, name):
    """vector / indexed / indexed_block / hindexed over old types whose extent differs
    from their size (resized, padded structs; MPI-3.1 §4.1.2, the constructors the paper
    relies on [L14:c1262 §3]), and the transpose idiom -- whole streams, counts 1-3,
    ragged fragments, every kernel family the planner picks."""
    rng = np.random.default_rng(hash(name) % 1000)
    mk = {
        "vec_resized": lambda: (("vector", 3000, 1, 3, _R8), 0, 3000 * 24 + 64),
        "idx_struct": lambda: (("indexed", [1, 2, 1] * 700, list(range(0, 2800 * 3, 4)), _SDI), 0, 2800 * 3 * 16 + 64),
        "iblk_resized": lambda: (("indexed_block", 2, list(range(0, 4000 * 5, 5)), _R8), 0, 4000 * 5 * 8 + 64),
        "vec_struct16": lambda: (("vector", 2000, 3, 5, _SHB), 0, 2000 * 5 * 4 + 64),
        "hidx_struct": lambda: (("hindexed", [2, 1] * 600, list(range(0, 1200 * 100, 100)), _SDI), 0, 1200 * 100 + 64),
        "transpose64": lambda: _transpose(64),
        "transpose300": lambda: _transpose(300),
    }
    rec, org, parent = mk[name]()
    ot = oracle.from_recipe(rec)
    size, ext = ot.size, ot.extent
    check_pack_unpack(torch_cuda, rec, org, parent)
    for count in (2, 3):
        total = count * size
        a, b = sorted(int(x) for x in rng.integers(0, total + 1, size=2))
        check_or_overlap(torch_cuda, rec, org, parent + (count - 1) * abs(ext) + 64, count, pos=a, nbytes=b - a,
                         origin_pad=int(rng.integers(0, 16)))


def test_transpose_idiom_equals_numpy(torch_cuda):
    """Transpose idiom on the GPU against numpy's transpose of the same bytes (an
    independent library routine): pack(contiguous(N, resized(vector(N,1,N)))) of a
    column-major A == A.T raveled column-major."""
    import torch
    from paper_conf_hpdc_wubvjd16_b200 import dt
    n = 257
    rec, org, parent = _transpose(n)
    src_h = fill_bytes(parent, 0x7A)
    A = src_h.view(np.float64).reshape(n, n).T      # A[r, c], column-major storage
    exp = np.ascontiguousarray(A.T).ravel(order="F").view(np.uint8)
    t = dt.from_recipe(rec).commit()
    out = torch.empty(len(exp), dtype=torch.uint8, device="cuda")
    dt.pack(t, 1, _dev(torch, src_h), out)
    torch.cuda.synchronize()
    assert np.array_equal(out.cpu().numpy(), exp)


@pytest.mark.parametrize("recipe", [("vector", 5, 2, 3, ("basic", "INT32")), _SDI,
                                    ("indexed", [0, 0], [1, 2], ("basic", "DOUBLE")),
                                    ("contiguous", 0, ("basic", "BYTE"))],
                         ids=["vector", "struct", "size0_indexed", "size0_contig"])
def test_count_or_size_zero(torch_cuda, recipe):
    """count 0, size 0 and pos beyond the stream: DT_OK, 0 bytes, destination untouched."""
    check_empty(torch_cuda, recipe, 0)
    check_empty(torch_cuda, recipe, 0, nbytes=0)
    check_empty(torch_cuda, recipe, 2, pos=1 << 20)


# ------------------------------------------------------------------ f2: pipelined first use
@pytest.mark.parametrize("first", ["pack", "unpack"])
@pytest.mark.parametrize("seed", [0, 1])
def test_pipelined_first_pack(torch_cuda, first, seed, monkeypatch):
    """f2: a huge irregular block list is flattened by its first whole-stream pack, in
    chunks pipelined with uploads, device scans and block-window packs of each
    finished range ([L18:c1121]-[L18:c1649 §3.2]).  Small thresholds force it on a
    120k-entry list with many zero gaps (merges across chunk boundaries, batches that
    end inside a block); the stream must equal the oracle's, the cached second pack
    too, and an unpack as first use must take the ordinary path."""
    import torch
    from paper_conf_hpdc_wubvjd16_b200 import dt
    monkeypatch.setenv("DT_PIPE_MIN", "1000")
    monkeypatch.setenv("DT_PIPE_CHUNK", "7001")
    monkeypatch.setenv("DT_FLATTEN", "pipe")
    rng = np.random.default_rng(40 + seed)
    n = 120_000
    lens = rng.integers(1, 17, size=n) * (4 if seed == 0 else 1)
    gaps = rng.integers(0, 4, size=n) * (4 if seed == 0 else 3)
    d = np.concatenate([[0], np.cumsum(lens + gaps)[:-1]]) + 64
    rec = ("hindexed", lens, d, ("basic", "BYTE"))
    parent = int(d[-1] + lens[-1] + 128)
    org = seed * 3  # misaligned origin for seed 1
    ot = oracle.from_recipe(rec)
    src_h = fill_bytes(parent + 16, 77 + seed)
    exp = oracle.pack(ot, 1, src_h, org)
    t = dt.from_recipe(rec).commit()
    src = _dev(torch, src_h)
    out = _poisoned(torch, len(exp))
    if first == "unpack":
        dst = torch.full((parent + 16,), 0xA5, dtype=torch.uint8, device="cuda")
        dt.unpack(t, 1, _dev(torch, exp), dst, origin_offset=org)
        ref = np.full(parent + 16, 0xA5, dtype=np.uint8)
        oracle.unpack(ot, 1, exp, ref, org)
        torch.cuda.synchronize()
        assert np.array_equal(dst.cpu().numpy(), ref)
    for _ in range(2):  # first (pipelined when `first` is pack) and cached
        dt.pack(t, 1, src, out.data_ptr() + GUARD, origin_offset=org)
        torch.cuda.synchronize()
        o = out.cpu().numpy()
        assert np.all(o[:GUARD] == 0xA5) and np.all(o[GUARD + len(exp):] == 0xA5)
        assert np.array_equal(o[GUARD:GUARD + len(exp)], exp)
    # the installed form is the ordinary one
    bd, bl = t.flatten(1)
    assert int(bl.sum()) == len(exp)


# ------------------------------------------------------------------ f2: GPU-side flattening
def _oracle_blocks(ot):
    """Merged block list of a BYTE-element typemap: runs of consecutive byte addresses, in
    typemap order (the flattening's definition, computed from the oracle's typemap)."""
    _, d = ot.typemap()
    if len(d) == 0:
        return d, d
    starts = np.concatenate([[0], np.flatnonzero(np.diff(d) != 1) + 1])
    lens = np.diff(np.concatenate([starts, [len(d)]]))
    return d[starts], lens


@pytest.mark.parametrize("case", ["sorted", "shuffled", "negative", "zeros", "all_adjacent"])
def test_gpu_flatten(torch_cuda, case, monkeypatch):
    """f2: dt_commit of a huge block list (an hindexed list of BYTE with per-entry
    counts) flattens it ON THE DEVICE (tile sums, scans, head emission, facts); the
    merged list (downloaded by dt_flatten), pack, unpack, the launch plan and the form
    facts must equal the oracle's / the host flattening's.  Cases: sorted with zero gaps
    (merges, also across 1024-entry tiles), shuffled entries (not sorted: unpack legality
    needs the host proof), negative displacements with a misaligned origin, entries of
    count 0 (the host flattening takes over), every entry adjacent (one block)."""
    import torch
    from paper_conf_hpdc_wubvjd16_b200 import dt
    monkeypatch.setenv("DT_PIPE_MIN", "1000")
    rng = np.random.default_rng({"sorted": 1, "shuffled": 2, "negative": 3, "zeros": 4, "all_adjacent": 5}[case])
    n = 50_000
    lens = rng.integers(1, 17, size=n) * 4
    gaps = rng.integers(0, 4, size=n) * 4
    if case == "all_adjacent":
        gaps[:] = 0
    if case == "zeros":
        lens[rng.integers(0, n, size=50)] = 0
    d = np.concatenate([[0], np.cumsum(lens + gaps)[:-1]]).astype(np.int64)
    if case == "shuffled":
        perm = rng.permutation(n)
        lens, d = lens[perm], d[perm]
    org = 0
    if case == "negative":
        d = d - int(d[-1]) // 2
        org = int(-d.min()) + 3
    rec = ("hindexed", lens, d, ("basic", "BYTE"))
    parent = int((d + lens).max()) + org + 64
    ot = oracle.from_recipe(rec)
    ob, ol = _oracle_blocks(ot)
    t = dt.from_recipe(rec).commit()
    monkeypatch.setenv("DT_FLATTEN", "host")
    th = dt.from_recipe(rec).commit()
    monkeypatch.delenv("DT_FLATTEN")
    # launch plans and form facts equal the host flattening's (before any download)
    fi, fh = t.form(), th.form()
    assert (fi.nblocks, fi.tsize, fi.granularity) == (fh.nblocks, fh.tsize, fh.granularity) == (len(ob), ot.size,
                                                                                                fh.granularity)
    for addr, pk in ((0x10000, 0x20000), (0x10003, 0x20000), (0x10000, 0x20008)):
        assert t.plan(1, addr, pk, 0, ot.size) == th.plan(1, addr, pk, 0, ot.size)
    src_h = fill_bytes(parent, 91)
    exp = oracle.pack(ot, 1, src_h, org)
    src = _dev(torch, src_h)
    out = _poisoned(torch, len(exp))
    dt.pack(t, 1, src, out.data_ptr() + GUARD, origin_offset=org)
    torch.cuda.synchronize()
    o = out.cpu().numpy()
    assert np.all(o[:GUARD] == 0xA5) and np.all(o[GUARD + len(exp):] == 0xA5)
    assert np.array_equal(o[GUARD:GUARD + len(exp)], exp)
    dst = torch.full((parent,), 0xA5, dtype=torch.uint8, device="cuda")
    dt.unpack(t, 1, _dev(torch, exp), dst, origin_offset=org)
    ref = np.full(parent, 0xA5, dtype=np.uint8)
    oracle.unpack(ot, 1, exp, ref, org)
    torch.cuda.synchronize()
    assert np.array_equal(dst.cpu().numpy(), ref)
    # a fragment (partial range: the launch plan needs the block prefix on the host)
    p0, p1 = len(exp) // 3 + 5, 2 * len(exp) // 3 + 1
    out.fill_(0xA5)
    dt.pack(t, 1, src, out.data_ptr() + GUARD, pos=p0, nbytes=p1 - p0, origin_offset=org)
    torch.cuda.synchronize()
    assert np.array_equal(out.cpu().numpy()[GUARD:GUARD + p1 - p0], exp[p0:p1])
    bd, bl = t.flatten(1)
    assert np.array_equal(bd, ob) and np.array_equal(bl, ol)
