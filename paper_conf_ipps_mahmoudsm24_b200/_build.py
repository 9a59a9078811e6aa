"""Build liblbmr.so in-tree with nvcc for sm_100a (no JIT, no torch extension)."""
from __future__ import annotations

import os
import shutil
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
LIBDIR = os.path.join(HERE, "_lib")
LIB = os.path.join(LIBDIR, "liblbmr.so")
SOURCES = ["capi.cpp", "grid_builder.cpp", "level_step.cu"]
HEADERS = ["kernels.h", "lattice.h", "grid_builder.h"]
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def nvcc() -> str:
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", shutil.which("nvcc")):
        if c and os.path.exists(c):
            return c
    raise RuntimeError("nvcc not found")


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = [os.path.join(CSRC, s) for s in SOURCES + HEADERS]
    deps.append(os.path.join(HERE, "..", "include", "lbmr.h"))
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False, out: str = None, defines=()) -> str:
    lib = out or LIB
    if not force and out is None and not _stale():
        return LIB
    os.makedirs(LIBDIR, exist_ok=True)
    objs = []
    for s in SOURCES:
        src = os.path.join(CSRC, s)
        obj = os.path.join(LIBDIR, s + ".o")
        cmd = [nvcc(), "-O3", "-std=c++17", *ARCH, "-lineinfo", "-Xcompiler", "-fPIC,-fopenmp,-O3",
               "-I", os.path.join(HERE, "..", "include"), *[f"-D{d}" for d in defines], "-c", src, "-o", obj]
        if s.endswith(".cu"):
            cmd += ["-Xptxas", "-v"] if verbose else []
        subprocess.check_call(cmd)
        objs.append(obj)
    tmp = lib + ".tmp"
    subprocess.check_call([nvcc(), "-shared", *ARCH, "-o", tmp, *objs, "-Xcompiler", "-fopenmp", "-lgomp"])
    os.replace(tmp, lib)
    for o in objs:
        os.remove(o)
    return lib


ALT_LIB = os.path.join(LIBDIR, "liblbmr_alt.so")


def build_alt(force: bool = False) -> str:
    """Diagnostic build for the fp32 rounding-floor checks (tools/fp32_floor.py,
    tests/test_gpu_parity.py): the same sources with the BGK step evaluated
    in another, equally valid association (LBMR_BGK_ALT_FORM=1).  Never loaded
    by the product path."""
    if force or not os.path.exists(ALT_LIB) or os.path.getmtime(ALT_LIB) < os.path.getmtime(LIB):
        build(out=ALT_LIB, defines=["LBMR_BGK_ALT_FORM=1"])
    return ALT_LIB


if __name__ == "__main__":
    print(build(force=True, verbose=True))
    print(build_alt(force=True))
