"""Seeded synthetic inputs and workload recipes, shared by tests, bench and smoke.

This module holds NONE of the method's arithmetic: it only (a) fills byte
buffers with seeded pseudo-random words and (b) states the constructor
arguments of the paper's workloads as plain nested tuples ("recipes").  The
oracle (``oracle/``) and the product library (``paper_conf_hpdc_wubvjd16_b200``)
each interpret a recipe with their OWN constructors; neither imports the other.

Recipe grammar (constructor name first, MPI-3.1 §4.1 argument order):
    ("basic", "DOUBLE")
    ("contiguous", n, R)
    ("vector", count, blocklen, stride_elems, R)     ("hvector", ..., stride_bytes, R)
    ("indexed", blocklens, displs_elems, R)          ("hindexed", blocklens, displs_bytes, R)
    ("indexed_block", blocklen, displs_elems, R)     ("hindexed_block", blocklen, displs_bytes, R)
    ("struct", blocklens, displs_bytes, [R...])
    ("subarray", sizes, subsizes, starts, "C"|"F", R)
    ("resized", R, lb, extent)

Input recipe (SURVEY §8(d) "Concrete synthetic inputs"): 8-byte word i of a
source buffer = splitmix64(seed XOR i) (random bit patterns incl. NaN/Inf
doubles, so only byte-exact movement passes); destinations are poisoned 0xA5.
Default seed 0x5EED0000 + config id.  KB/MB/GB = 2^10/2^20/2^30 (reading A20).
"""
from __future__ import annotations

import math

import numpy as np

POISON = 0xA5
MASK64 = (1 << 64) - 1


def splitmix64(x: np.ndarray) -> np.ndarray:
    """Vectorised splitmix64 finaliser over uint64 (Steele, Lea, Flood 2014)."""
    with np.errstate(over="ignore"):
        z = x + np.uint64(0x9E3779B97F4A7C15)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        return z ^ (z >> np.uint64(31))


def fill_bytes(nbytes: int, seed: int, chunk_words: int = 1 << 24) -> np.ndarray:
    """uint8 buffer whose 8-byte word i = splitmix64(seed ^ i) (little-endian)."""
    nw = (nbytes + 7) // 8
    out = np.empty(nw, dtype=np.uint64)
    s = np.uint64(seed & MASK64)
    for w0 in range(0, nw, chunk_words):
        w1 = min(nw, w0 + chunk_words)
        out[w0:w1] = splitmix64(np.arange(w0, w1, dtype=np.uint64) ^ s)
    return out.view(np.uint8)[:nbytes]


def poison(nbytes: int) -> np.ndarray:
    return np.full(nbytes, POISON, dtype=np.uint8)


def address_words(nbytes: int) -> np.ndarray:
    """Address-encoding source: each aligned u32 word holds its own byte offset
    (so a pack of 4-byte-aligned elements outputs the list of source addresses)."""
    nw = (nbytes + 3) // 4
    return (np.arange(nw, dtype=np.uint32) * np.uint32(4)).view(np.uint8)[:nbytes].copy()


def seed_for(config_id: int) -> int:
    return 0x5EED0000 + config_id


# ---------------------------------------------------------------- workloads
D = ("basic", "DOUBLE")
F32 = ("basic", "FLOAT")
I32 = ("basic", "INT32")


def c1_submatrix(n_sub: int = 256, lda: int = 1024, r0: int = 0, c0: int = 0):
    """C1 / W1 "V": n_sub x n_sub double sub-matrix of a column-major matrix with
    leading dimension lda: one column per block, stride = lda (PAPER.md
    [L22:c1966 §5.1]).  Returns (recipe, origin_byte_offset, parent_bytes)."""
    return ("vector", n_sub, n_sub, lda, D), (c0 * lda + r0) * 8, lda * lda * 8


def c2_lower_triangle(n: int = 4096):
    """C2 / W2 "T": lower triangle (diagonal included) of a column-major n x n
    double matrix; column j holds n-j elements starting at row j, i.e. element
    displacement j*(n+1) (PAPER.md [L22:c2839 §5.1]; reading A2)."""
    bl = [n - j for j in range(n)]
    dp = [j * (n + 1) for j in range(n)]
    return ("indexed", bl, dp, D), 0, n * n * 8


def upper_triangle(n: int):
    """Upper triangle incl. diagonal: column j holds rows 0..j (reading A2)."""
    return ("indexed", [j + 1 for j in range(n)], [j * n for j in range(n)], D), 0, n * n * 8


def stair_triangle(n: int, nb: int):
    """T-stair (Fig. 5, [L24:c496 §5.1]; reading A4): column j has n - nb*floor(j/nb)
    elements from row nb*floor(j/nb)."""
    bl = [n - nb * (j // nb) for j in range(n)]
    dp = [j * n + nb * (j // nb) for j in range(n)]
    return ("indexed", bl, dp, D), 0, n * n * 8


def c3_block_cyclic(n: int = 8192, nb: int = 64, p: int = 0, q: int = 1):
    """C3: blocks owned by process (p,q) of a 2x2 virtual grid in a column-major
    n x n double matrix with block size nb ("basic blocks of the ScaLAPACK data
    manipulation", [L22:c1714]; reading A18).  Origin = element (p*nb, q*nb)."""
    nblk = n // (2 * nb)
    inner = ("vector", nblk, nb, 2 * nb, D)                # row blocks of one column
    cols = ("hvector", nb, 1, n * 8, inner)               # nb consecutive columns
    rec = ("hvector", nblk, 1, 2 * nb * n * 8, cols)      # every other column block
    return rec, (q * nb * n + p * nb) * 8, n * n * 8


HALO_FACES = ("x-", "x+", "y-", "y+", "z-", "z+")


def c4_face(face: str, n: int = 512, h: int = 1, ghost: bool = False):
    """C4: one face of a C-ordered A[z][y][x] float array of (n+2h)^3 (interior
    [h, n+h)^3) as a subarray (reading A17).  ghost=False: the interior boundary
    layer that is sent; ghost=True: the ghost layer that is received."""
    L = n + 2 * h
    dim = {"z": 0, "y": 1, "x": 2}[face[0]]
    sub = [n, n, n]
    st = [h, h, h]
    sub[dim] = h
    if face[1] == "-":
        st[dim] = 0 if ghost else h
    else:
        st[dim] = n + h if ghost else n
    return ("subarray", [L, L, L], sub, st, "C", F32), 0, L * L * L * 4


PARTICLE = ("resized", ("struct", [1, 3, 3, 1], [0, 8, 32, 56],
                        [I32, D, D, F32]), 0, 64)


def c5_particles(message_bytes: int, seed: int = 1234):
    """C5: LAMMPS-style index list ([L14:c2154 §3]; reading A19) —
    hindexed_block(nsel, 1, idx*64, particle) with idx a sorted Bernoulli(0.5)
    subset; nsel = ceil(m/56)."""
    nsel = max(1, math.ceil(message_bytes / 56))
    rng = np.random.default_rng(seed)
    # draw enough candidates, keep the first nsel selected ones
    cand = 2 * nsel + 64
    keep = np.flatnonzero(rng.random(cand) < 0.5)
    while len(keep) < nsel:
        cand *= 2
        keep = np.flatnonzero(np.random.default_rng(seed).random(cand) < 0.5)
    idx = keep[:nsel].astype(np.int64)
    parent = (int(idx[-1]) + 1) * 64
    return ("hindexed_block", 1, idx * 64, PARTICLE), 0, parent


def c5b_irregular(message_bytes: int, seed: int = 42):
    """C5b: hindexed over BYTE with random lengths in {4..64 step 4} and random
    gaps in {0..60 step 4} (reading A19)."""
    rng = np.random.default_rng(seed)
    est = max(1, message_bytes // 34 + 16)
    lens = rng.integers(1, 17, size=est, dtype=np.int64) * 4
    gaps = rng.integers(0, 16, size=est, dtype=np.int64) * 4
    cs = np.cumsum(lens)
    nb = int(np.searchsorted(cs, message_bytes) + 1)
    nb = min(nb, est)
    lens = lens[:nb].copy()
    lens[-1] -= max(0, int(cs[nb - 1]) - message_bytes)
    lens = lens[lens > 0]
    gaps = gaps[: len(lens)]
    disp = np.concatenate([[0], np.cumsum(lens[:-1] + gaps[:-1])]).astype(np.int64)
    parent = int(disp[-1] + lens[-1]) if len(lens) else 0
    return ("hindexed", lens, disp, ("basic", "BYTE")), 0, parent


CONFIGS = {
    "C1": lambda: c1_submatrix(),
    "C1b": lambda: c1_submatrix(r0=1, c0=1),
    "C2": lambda: c2_lower_triangle(),
    "C3": lambda: c3_block_cyclic(),
    "C4x": lambda: c4_face("x-"),
    "C4y": lambda: c4_face("y-"),
    "C4z": lambda: c4_face("z-"),
    "C5": lambda: c5_particles(1 << 20),
}
