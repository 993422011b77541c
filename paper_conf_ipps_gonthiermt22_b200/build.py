"""Build libdts.so in-tree for sm_100a (nvcc cross-compiles without a GPU)."""
from __future__ import annotations

import glob
import os
import subprocess

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "lib", "libdts.so")
LIB_PROF = os.path.join(PKG, "lib", "libdts_prof.so")  # per-phase cycle probes (-DDTS_PROF)
INCLUDE = os.path.join(ROOT, "include")

NVCC_FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
              "-Xcompiler", "-fPIC", "-shared", "-Xptxas", "-O3"]


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def _stale(lib: str = LIB) -> bool:
    if not os.path.exists(lib):
        return True
    t = os.path.getmtime(lib)
    deps = sources() + glob.glob(os.path.join(CSRC, "*.cuh")) + [os.path.join(INCLUDE, "dts.h")]
    return any(os.path.getmtime(p) > t for p in deps)


def _build_one(lib: str, extra, force: bool, verbose: bool) -> None:
    if not force and not _stale(lib):
        return
    os.makedirs(os.path.dirname(lib), exist_ok=True)
    nvcc = os.environ.get("NVCC", "nvcc")
    cmd = [nvcc, *NVCC_FLAGS, *extra, "-I", INCLUDE, "-o", lib + ".tmp", *sources()]
    if verbose:
        print(" ".join(cmd))
    subprocess.check_call(cmd)
    os.replace(lib + ".tmp", lib)


def build(force: bool = False, verbose: bool = False) -> str:
    """Build lib/libdts.so (the product) and lib/libdts_prof.so (the same
    kernels with per-phase cycle probes, loaded when DTS_PROFILE=1)."""
    _build_one(LIB, [], force, verbose)
    _build_one(LIB_PROF, ["-DDTS_PROF"], force, verbose)
    return LIB


if __name__ == "__main__":
    print(build(force=True, verbose=True))
