"""Build libdt.so in-tree with nvcc for sm_100a (no JIT cache, no torch extension).

The library is plain C-ABI (include/dt.h); the Python binding loads it with
ctypes.  cudart is linked statically; NCCL is dlopen()ed at dt_comm_init time.
"""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIBDIR = os.path.join(HERE, "lib")
LIB = os.path.join(LIBDIR, "libdt.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
SOURCES = ["dt_types.cpp", "dt_kernels.cu", "dt_xfer.cu", "dt_direct.cu"]


def _sources():
    return [os.path.join(CSRC, s) for s in SOURCES if os.path.exists(os.path.join(CSRC, s))]


def _deps():
    out = _sources() + [os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith((".h", ".cuh"))]
    out.append(os.path.join(ROOT, "include", "dt.h"))
    out.append(os.path.abspath(__file__))
    return out


def needs_build() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(p) > t for p in _deps())


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not needs_build():
        return LIB
    os.makedirs(LIBDIR, exist_ok=True)
    objs, cmds = [], []
    headers = [p for p in _deps() if not p.endswith((".cu", ".cpp"))]
    flags_file = os.path.join(LIBDIR, "flags.txt")
    flags = os.environ.get("DT_NVCC_FLAGS", "") + "|" + os.environ.get("DT_PTXAS_V", "")
    same_flags = os.path.exists(flags_file) and open(flags_file).read() == flags
    for src in _sources():
        obj = os.path.join(LIBDIR, os.path.basename(src) + ".o")
        objs.append(obj)
        # per-object rebuild: its source, any header or this script newer than the object
        if (not force and same_flags and os.path.exists(obj)
                and all(os.path.getmtime(p) <= os.path.getmtime(obj) for p in [src, *headers])):
            continue
        cmd = [NVCC, *ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-O3",
               "-I", os.path.join(ROOT, "include"), "-c", src, "-o", obj]
        if src.endswith(".cpp"):
            cmd[1:1] = ["-x", "cu"]
        if os.environ.get("DT_PTXAS_V"):
            cmd += ["-Xptxas", "-v"]
        if os.environ.get("DT_NVCC_FLAGS"):  # tuning experiments, e.g. -DDT_STORE_WB=1
            cmd += os.environ["DT_NVCC_FLAGS"].split()
        if verbose:
            print(" ".join(cmd), file=sys.stderr)
        cmds.append(cmd)
    # translation units are independent: compile them concurrently
    from concurrent.futures import ThreadPoolExecutor
    with ThreadPoolExecutor(max_workers=len(cmds) or 1) as ex:
        list(ex.map(subprocess.check_call, cmds))
    with open(flags_file, "w") as fh:
        fh.write(flags)
    tmp = LIB + f".tmp{os.getpid()}"
    cmd = [NVCC, *ARCH, "-shared", "-cudart", "static", "-o", tmp, *objs, "-ldl", "-lpthread", "-lrt"]
    if verbose:
        print(" ".join(cmd), file=sys.stderr)
    subprocess.check_call(cmd)
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
