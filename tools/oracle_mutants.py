"""Mutation check of the oracle's pins (tests/test_oracle_pins.py).

Copies oracle/, workloads/ and the pin tests into a scratch directory, applies
one deliberate bug at a time to oracle/oracle.c, rebuilds it and runs the pins.
Every mutant must make at least one pin fail; a surviving mutant is a pin gap.
Usage: python tools/oracle_mutants.py   (CPU only, ~1 min)
"""
import os
import shutil
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

# (name, original text, mutated text) in oracle/oracle.c
MUTANTS = [
    ("vector stride by size(old)",
     "return or_hvector(count, blocklen, stride * ext(old), old);",
     "return or_hvector(count, blocklen, stride * old->size, old);"),
    ("indexed displs by size(old)",
     "for (int64_t i = 0; i < count; i++) db[i] = d[i] * ext(old);",
     "for (int64_t i = 0; i < count; i++) db[i] = d[i] * old->size;"),
    ("struct eps fixed 8",
     "int64_t r = ((e % a->align) + a->align) % a->align;\n    if (r) t->ub += a->align - r;",
     "int64_t r = ((e % 8) + 8) % 8;\n    if (r) t->ub += 8 - r;"),
    ("no struct eps",
     "if (r) t->ub += a->align - r;",
     "(void)r;"),
    ("hvector drops j*extent",
     "bacc_copy(&a, old, i * stride + j * ext(old));",
     "bacc_copy(&a, old, i * stride);"),
    ("hindexed j*size",
     "bacc_copy(&a, old, dps[i] + j * ext(old));",
     "bacc_copy(&a, old, dps[i] + j * old->size);"),
    ("contiguous at i*size",
     "for (int64_t i = 0; i < count; i++) bacc_copy(&a, old, i * ext(old));",
     "for (int64_t i = 0; i < count; i++) bacc_copy(&a, old, i * old->size);"),
    # the typemap walk (what pack/unpack move)
    ("walk: contiguous at i*size",
     "for (int64_t i = 0; i < t->count && !v->done; i++) walk(t->old, shift + i * ext(t->old), v);",
     "for (int64_t i = 0; i < t->count && !v->done; i++) walk(t->old, shift + i * t->old->size, v);"),
    ("walk: hvector drops j*extent",
     "walk(t->old, shift + i * t->stride + j * ext(t->old), v);",
     "walk(t->old, shift + i * t->stride + j * t->old->size, v);"),
    ("walk: hindexed j*size",
     "walk(t->old, shift + t->dps[i] + j * ext(t->old), v);",
     "walk(t->old, shift + t->dps[i] + j * t->old->size, v);"),
    ("walk: struct j*size",
     "walk(t->types[i], shift + t->dps[i] + j * ext(t->types[i]), v);",
     "walk(t->types[i], shift + t->dps[i] + j * t->types[i]->size, v);"),
    ("walk: subarray Fortran order as C",
     "    for (int d = t->ndims - 1; d >= 0; d--) lin = lin * t->sizes[d] + (t->starts[d] + idx[d]);",
     "    for (int d = 0; d < t->ndims; d++) lin = lin * t->sizes[d] + (t->starts[d] + idx[d]);"),
    ("walk: subarray ignores starts",
     "    for (int d = 0; d < t->ndims; d++) lin = lin * t->sizes[d] + (t->starts[d] + idx[d]);\n  } else {",
     "    for (int d = 0; d < t->ndims; d++) lin = lin * t->sizes[d] + idx[d];\n  } else {"),
    ("walk: instance k at k*size",
     "  for (int64_t k = 0; k < count && !v->done; k++) walk(t, k * ext(t), v);\n}",
     "  for (int64_t k = 0; k < count && !v->done; k++) walk(t, k * t->size, v);\n}"),
    ("walk: resume seeks instances by extent",
     "    int64_t k0 = v->pos / t->size;",
     "    int64_t k0 = v->pos / (ext(t) > 0 ? ext(t) : t->size);"),
    ("unpack ignores pos",
     "    if (p >= v->pos && p < v->end) v->dst[disp + b] = v->src[p - v->pos];",
     "    if (p >= v->pos && p < v->end) v->dst[disp + b] = v->src[p];"),
    ("pack writes at the stream position",
     "    if (p >= v->pos && p < v->end) v->dst[p - v->pos] = v->src[disp + b];",
     "    if (p >= v->pos && p < v->end) v->dst[p] = v->src[disp + b];"),
    # bounds (MPI-3.1 §4.1.6, §4.1.7)
    ("resized keeps the old lb",
     "  t->lb = lb; t->ub = lb + extent; t->has_lb = 1; t->has_ub = 1;",
     "  t->lb = old->lb; t->ub = old->lb + extent; t->has_lb = 1; t->has_ub = 1;"),
    ("markers ignored (data bounds only)",
     "  t->lb = a->any_lbm ? a->lbm : (a->any_data ? a->dlb : 0);",
     "  t->lb = a->any_data ? a->dlb : (a->any_lbm ? a->lbm : 0);"),
    ("true_ub from the extent",
     "  t->true_ub = a->any_data ? a->tub : 0;",
     "  t->true_ub = a->any_data ? t->ub : 0;"),
    ("subarray extent = box size",
     "  t->lb = 0; t->ub = tot * ext(old); t->has_lb = 1; t->has_ub = 1;",
     "  t->lb = 0; t->ub = nel * ext(old); t->has_lb = 1; t->has_ub = 1;"),
]


def run_one(tmp, name, a, b):
    src = os.path.join(tmp, "oracle", "oracle.c")
    orig = open(os.path.join(ROOT, "oracle", "oracle.c")).read()
    if a not in orig:
        return name, "NOT APPLIED (pattern not found)"
    open(src, "w").write(orig.replace(a, b))
    lib = os.path.join(tmp, "oracle", "liboracle.so")
    if os.path.exists(lib):
        os.remove(lib)
    # (the meta-test that runs this tool is deselected: inside the scratch copy it would
    # fail for every mutant and report them all killed)
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-p", "no:cacheprovider",
                        "-k", "not mutants_killed", os.path.join(tmp, "tests", "test_oracle_pins.py")],
                       cwd=tmp, capture_output=True, text=True)
    return name, "killed" if r.returncode != 0 else "SURVIVED"


def main():
    tmp = tempfile.mkdtemp(prefix="omut")
    try:
        for d in ("oracle", "workloads"):
            shutil.copytree(os.path.join(ROOT, d), os.path.join(tmp, d),
                            ignore=shutil.ignore_patterns("*.so", "__pycache__"))
        os.makedirs(os.path.join(tmp, "tests"))
        for f in ("__init__.py", "conftest.py", "test_oracle_pins.py"):
            shutil.copy(os.path.join(ROOT, "tests", f), os.path.join(tmp, "tests", f))
        shutil.copytree(os.path.join(ROOT, "tests", "golden"), os.path.join(tmp, "tests", "golden"))
        bad = 0
        name, res = run_one(tmp, "unmutated (must pass)", "", "")
        print(f"{'ok' if res == 'SURVIVED' else 'BROKEN':10s} {name}")
        bad += res != "SURVIVED"
        for m in MUTANTS:
            name, res = run_one(tmp, *m)
            print(f"{res:10s} {name}")
            bad += res != "killed"
        return 1 if bad else 0
    finally:
        shutil.rmtree(tmp, ignore_errors=True)


if __name__ == "__main__":
    sys.exit(main())
