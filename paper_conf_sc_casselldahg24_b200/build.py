"""Build the sm_100a shared library libnbody_b200.so in-tree with nvcc.

The library is the product: every stage of the step runs in its kernels.
Usage: python -m paper_conf_sc_casselldahg24_b200.build [--force] [--verbose]
"""
from __future__ import annotations

import glob
import os
import shutil
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libnbody_b200.so")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _nvcc() -> str:
    for cand in (shutil.which("nvcc"), "/usr/local/cuda/bin/nvcc"):
        if cand and os.path.exists(cand):
            return cand
    raise RuntimeError("nvcc not found: the CUDA toolkit is required to build libnbody_b200.so")


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def _deps():
    return sources() + sorted(glob.glob(os.path.join(CSRC, "*.cuh"))) + [os.path.join(ROOT, "include", "nbody.h"),
                                                                          os.path.abspath(__file__)]


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(p) > t for p in _deps())


def nccl_dir():
    """The NCCL the torch wheel ships (nvidia/nccl/{include,lib}), or None."""
    for p in sys.path:
        d = os.path.join(p, "nvidia", "nccl")
        if os.path.exists(os.path.join(d, "include", "nccl.h")) and os.path.isdir(os.path.join(d, "lib")):
            return d
    return None


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not stale():
        return LIB
    # several processes (torchrun ranks, pytest workers) may find the library
    # stale at once: one builds under an exclusive lock, the others wait and
    # then find it fresh; the result is written under a per-process name and
    # renamed into place atomically
    import fcntl
    with open(LIB + ".lock", "w") as lock:
        fcntl.flock(lock, fcntl.LOCK_EX)
        try:
            if not force and not stale():
                return LIB
            return _build_locked(verbose)
        finally:
            fcntl.flock(lock, fcntl.LOCK_UN)


def _build_locked(verbose: bool) -> str:
    nccl = []
    d = nccl_dir()
    if d:
        lib = os.path.join(d, "lib")
        so = sorted(f for f in os.listdir(lib) if f.startswith("libnccl.so"))
        nccl = ["-DNBODY_WITH_NCCL", "-I", os.path.join(d, "include"), "-L", lib, f"-l:{so[0]}",
                "-Xlinker", f"-rpath,{lib}"]
    extra = os.environ.get("NBODY_NVCC_FLAGS", "").split()  # tuning experiments only
    tmp = f"{LIB}.{os.getpid()}.tmp"
    cmd = [_nvcc(), *ARCH, "-O3", "-lineinfo", "-std=c++17", "-shared", "-Xcompiler", "-fPIC",
           "-I", os.path.join(ROOT, "include"), *nccl, *extra, "-o", tmp, *sources()]
    if verbose:
        cmd.insert(1, "-Xptxas=-v")
        print(" ".join(cmd), file=sys.stderr)
    subprocess.run(cmd, check=True)
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose="--verbose" in sys.argv)
    print(LIB)
