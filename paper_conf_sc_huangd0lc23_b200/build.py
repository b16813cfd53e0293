"""Builds libcuszp.so in-tree with nvcc for sm_100a (B200).

Flags pin bit-exactness: no FMA contraction
(-fmad=false; the kernels also use explicit __fmul_rn/__fadd_rn/__fmaf_rn),
IEEE division/sqrt, no FTZ, no fast math.  The CUDA runtime is linked
statically so the library does not depend on torch's libcudart.
"""
from __future__ import annotations

import glob
import os
import shutil
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libcuszp.so")

ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
NVCC_FLAGS = [
    "-O3", "-std=c++17", "-lineinfo", "-fmad=false", "-prec-div=true", "-prec-sqrt=true",
    "-ftz=false", "-Xcompiler", "-fPIC", "-Xcompiler", "-O2", "--cudart", "static",
    "-I", os.path.join(ROOT, "include"),
]


def nvcc() -> str:
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", shutil.which("nvcc")):
        if c and os.path.exists(c):
            return c
    raise RuntimeError("nvcc not found")


def sources() -> list[str]:
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def deps() -> list[str]:
    return sources() + glob.glob(os.path.join(CSRC, "*.cuh")) + [os.path.join(ROOT, "include", "cuszp.h"), __file__]


def needs_build() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(d) > t for d in deps())


def build(force: bool = False, verbose: bool = False, defines: list[str] | None = None,
          out: str | None = None) -> str:
    """Compile every csrc/*.cu into one shared library (default: the in-tree
    libcuszp.so).  ``defines``/``out`` build diagnostic variants elsewhere."""
    target = out or LIB
    if out is None and not force and not needs_build():
        return LIB
    cmd = [nvcc(), *ARCH, *NVCC_FLAGS, *[f"-D{d}" for d in (defines or [])], "-shared", "-o", target + ".tmp",
           *sources()]
    if verbose:
        cmd += ["-Xptxas", "-v"]
    subprocess.run(cmd, check=True)
    os.replace(target + ".tmp", target)
    return target


if __name__ == "__main__":
    print(build(force=True, verbose="-v" in sys.argv))
