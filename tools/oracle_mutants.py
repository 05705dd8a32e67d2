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
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-p", "no:cacheprovider",
                        os.path.join(tmp, "tests", "test_oracle_pins.py")],
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
        for m in MUTANTS:
            name, res = run_one(tmp, *m)
            print(f"{res:10s} {name}")
            bad += res != "killed"
        return 1 if bad else 0
    finally:
        shutil.rmtree(tmp, ignore_errors=True)


if __name__ == "__main__":
    sys.exit(main())
