"""Build liblzr.so in-tree with nvcc for sm_100a (no JIT cache, no torch
extension machinery: the library has a plain C ABI)."""
from __future__ import annotations

import glob
import os
import subprocess

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "liblzr.so")

NVCC_FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-O3", "-lineinfo", "-std=c++17",
    "-Xcompiler", "-fPIC", "-shared", "-cudart", "static",
    "-Xptxas", "-warn-spills",
]


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def deps():
    return sources() + sorted(glob.glob(os.path.join(CSRC, "*.cuh"))) + [
        os.path.join(ROOT, "include", "lzr.h")]


def source_hash(kernel: str = "encode") -> str:
    """Hash of the sources one kernel of liblzr.so is built from (encode.cu +
    the shared header + include/lzr.h for "encode"; every source for "all"):
    stamps ncu captures so that the bench drops profile-derived keys taken on
    a different build of that kernel (no toolchain needed to compute it)."""
    import hashlib

    files = deps() if kernel == "all" else [
        os.path.join(CSRC, f"{kernel}.cu"), os.path.join(CSRC, "lzr_internal.cuh"),
        os.path.join(ROOT, "include", "lzr.h")]
    h = hashlib.sha256()
    for d in files:
        h.update(os.path.basename(d).encode())
        with open(d, "rb") as f:
            h.update(f.read())
    return h.hexdigest()[:16]


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(d) > t for d in deps())


def build_timing() -> str:
    """Instrumented variant (per-phase cycle counters, tools/phase_times.py)."""
    out = os.path.join(PKG, "liblzr_timing.so")
    subprocess.check_call(["nvcc", *NVCC_FLAGS, "-DLZR_PHASE_TIMING", "-o", out, *sources()])
    return out


def build_watchdog() -> str:
    """Debug variant: spin loops trap with a message after ~2^26 iterations."""
    out = os.path.join(PKG, "liblzr_dbg.so")
    subprocess.check_call(["nvcc", *NVCC_FLAGS, "-DLZR_WATCHDOG", "-o", out, *sources()])
    return out


def build(force: bool = False, verbose: bool = False) -> str:
    if force or stale():
        cmd = ["nvcc", *NVCC_FLAGS, *(["-Xptxas", "-v"] if verbose else []),
               "-o", LIB + ".tmp", *sources()]
        subprocess.check_call(cmd)
        os.replace(LIB + ".tmp", LIB)
    return LIB


if __name__ == "__main__":
    import sys
    if "--timing" in sys.argv:
        print(build_timing())
    elif "--watchdog" in sys.argv:
        print(build_watchdog())
    else:
        build(force="-f" in sys.argv, verbose="-v" in sys.argv)
        print(LIB)
