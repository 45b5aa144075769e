"""Build the sm_100a shared library libbandlu.so in-tree (nvcc, no torch JIT)."""
from __future__ import annotations

import glob
import os
import subprocess

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
LIB = os.environ.get("BANDLU_LIB") or os.path.join(PKG, "libbandlu.so")  # override: experiment builds
SRC = os.path.join(PKG, "csrc", "bandlu.cu")

NVCC_FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-O3", "-lineinfo", "-std=c++17",
    "--fmad=false",          # no implicit contraction: FMA only where written (__fma_rn)
    "-prec-div=true", "-prec-sqrt=true", "-ftz=false",
    "-Xptxas", "-v",
    "-Xcompiler", "-fPIC", "-shared",
    "-I", os.path.join(ROOT, "include"),
]


def _nvcc() -> str:
    for c in ("/usr/local/cuda/bin/nvcc", "nvcc"):
        if os.path.isabs(c) and os.path.exists(c):
            return c
    return "nvcc"


def sources() -> list[str]:
    return sorted(glob.glob(os.path.join(PKG, "csrc", "*.cu")) + glob.glob(os.path.join(PKG, "csrc", "*.cuh"))
                  + glob.glob(os.path.join(ROOT, "include", "*.h")))


def needs_build() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(s) > t for s in sources())


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not needs_build():
        return LIB
    os.makedirs(os.path.join(ROOT, "build"), exist_ok=True)
    log = os.path.join(ROOT, "build", "ptxas.log")
    tmp = LIB + f".tmp{os.getpid()}"
    cmd = [_nvcc(), *NVCC_FLAGS, SRC, "-o", tmp]
    with open(log, "w") as f:
        r = subprocess.run(cmd, stdout=f, stderr=subprocess.STDOUT)
    if r.returncode != 0:
        raise RuntimeError("nvcc failed:\n" + open(log).read()[-6000:])
    os.replace(tmp, LIB)
    if verbose:
        print(open(log).read())
    return LIB


if __name__ == "__main__":
    import sys
    build(force="-f" in sys.argv, verbose="-v" in sys.argv)
    print(LIB)
