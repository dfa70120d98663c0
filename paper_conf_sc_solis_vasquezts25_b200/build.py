"""Build libad.so in-tree with nvcc for sm_100a (no JIT cache: the .so travels with the repo)."""
from __future__ import annotations

import os
import subprocess

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
SRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libad.so")
SOURCES = ["ad_api.cu"]
HEADERS = ["ad_internal.h", "ad_kernels.cuh"]

NVCC_FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-O3", "-lineinfo", "-std=c++17", "-ftz=true",
    # no multiply-add contraction, neither in NVVM (-fmad=false) nor in ptxas: every FMA
    # is an explicit fmaf / fma / fma.f32x2 of the source, so every kernel variant
    # (register budget, cherry-only twin, A14-instrumented) rounds identically and
    # results do not depend on which one a launch picks.  (ptxas fuses a packed
    # mul.f32x2 -> add/sub.f32x2 pair into FFMA2 even then: the packed code has none.)
    "-fmad=false", "-Xptxas", "--fmad=false",
    "-Xcompiler", "-fPIC", "-shared",
]


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = [os.path.join(SRC, f) for f in SOURCES + HEADERS] + [os.path.join(ROOT, "include", "ad.h")]
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False, extra: list[str] | None = None) -> str:
    if not force and not _stale():
        return LIB
    nvcc = os.environ.get("NVCC", "nvcc")
    cmd = [nvcc, *NVCC_FLAGS, *(extra or []), "-I", os.path.join(ROOT, "include"), "-o", LIB + ".tmp",
           *[os.path.join(SRC, f) for f in SOURCES]]
    if verbose:
        print(" ".join(cmd))
    subprocess.check_call(cmd)
    os.replace(LIB + ".tmp", LIB)
    return LIB


if __name__ == "__main__":
    print(build(force=True, verbose=True, extra=["-Xptxas", "-v"]))
