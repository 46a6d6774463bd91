"""Seeded synthetic write streams (input generator shared by tests, oracle
baseline and bench; holds none of the method's arithmetic).

``fill_host`` runs the C generator on host threads; ``fill_device`` runs the
identical generator (same source, synth_core.h) as a CUDA kernel so large
shards can be produced in place on each GPU.  Recipe: synth_core.h / DESIGN.md.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
HOST_LIB = os.path.join(_HERE, "libsynth.so")
CUDA_LIB = os.path.join(_HERE, "libsynth_cuda.so")

TEXT, RANDOM, ZERORUNS, MIX, CR2 = 0, 1, 2, 3, 4
DEDUP = 0x10  # flag: dedup-2.0 logical stream over the base class (synth_core.h)
CLASSES = {"text": TEXT, "random": RANDOM, "zeroruns": ZERORUNS, "mix": MIX, "cr2": CR2,
           "mix_dedup": MIX | DEDUP}
DEFAULT_SEED = 0x4C5A52

NVCC_ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _stale(target, deps):
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(d) > t for d in deps)


def build_host(force=False):
    deps = [os.path.join(_HERE, f) for f in ("synth_host.c", "synth_core.h")]
    if force or _stale(HOST_LIB, deps):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-Wall", "-fPIC", "-shared", "-pthread",
                               "-o", HOST_LIB + ".tmp", deps[0], "-lm"])
        os.replace(HOST_LIB + ".tmp", HOST_LIB)
    return HOST_LIB


def build_cuda(force=False):
    deps = [os.path.join(_HERE, f) for f in ("synth_cuda.cu", "synth_core.h")]
    if force or _stale(CUDA_LIB, deps):
        subprocess.check_call(["nvcc", *NVCC_ARCH, "-O3", "-lineinfo", "-shared",
                               "-Xcompiler", "-fPIC", "-cudart", "static",
                               "-o", CUDA_LIB + ".tmp", deps[0]])
        os.replace(CUDA_LIB + ".tmp", CUDA_LIB)
    return CUDA_LIB


_host = None
_cuda = None
_tables_cache: dict = {}


def _hlib():
    global _host
    if _host is None:
        build_host()
        L = ctypes.CDLL(HOST_LIB)
        L.syn_build_tables.argtypes = [ctypes.c_uint64, ctypes.c_void_p]
        L.syn_tables_bytes.restype = ctypes.c_size_t
        L.syn_fill.argtypes = [ctypes.c_void_p, ctypes.c_size_t, ctypes.c_uint32, ctypes.c_int,
                               ctypes.c_uint64, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_int]
        L.syn_chunk_class_of.argtypes = [ctypes.c_int, ctypes.c_uint64, ctypes.c_uint64]
        L.syn_dedup_source_of.argtypes = [ctypes.c_uint64, ctypes.c_uint64]
        L.syn_dedup_source_of.restype = ctypes.c_uint64
        _host = L
    return _host


def tables(seed: int = DEFAULT_SEED) -> np.ndarray:
    if seed not in _tables_cache:
        L = _hlib()
        buf = np.zeros(L.syn_tables_bytes(), np.uint8)
        L.syn_build_tables(seed, ctypes.c_void_p(buf.ctypes.data))
        _tables_cache[seed] = buf
    return _tables_cache[seed]


def dedup_source(chunk: int, seed: int = DEFAULT_SEED) -> int:
    """Fresh chunk whose content logical chunk `chunk` of a dedup stream carries."""
    return int(_hlib().syn_dedup_source_of(seed, chunk))


def chunk_class(cls: int, chunk: int, seed: int = DEFAULT_SEED) -> int:
    return _hlib().syn_chunk_class_of(cls, seed, chunk)


def fill_host(n: int, chunk_size: int = 4096, cls: int | str = MIX, seed: int = DEFAULT_SEED,
              first_chunk: int = 0, n_threads: int | None = None, out: np.ndarray | None = None):
    if isinstance(cls, str):
        cls = CLASSES[cls]
    if n_threads is None:
        n_threads = len(os.sched_getaffinity(0))
    if out is None:
        out = np.empty(max(1, n), np.uint8)
    t = tables(seed)
    st = _hlib().syn_fill(ctypes.c_void_p(out.ctypes.data), n, chunk_size, cls, seed, first_chunk,
                          ctypes.c_void_p(t.ctypes.data), n_threads)
    if st != 0:
        raise ValueError("syn_fill failed")
    return out[:n]


def fill_device(t, chunk_size: int = 4096, cls: int | str = MIX, seed: int = DEFAULT_SEED,
                first_chunk: int = 0, stream=None):
    """Fill a uint8 CUDA tensor in place (chunks first_chunk, first_chunk+1, ...)."""
    import torch

    global _cuda
    if isinstance(cls, str):
        cls = CLASSES[cls]
    if _cuda is None:
        build_cuda()
        L = ctypes.CDLL(CUDA_LIB)
        L.syn_fill_device.argtypes = [ctypes.c_void_p, ctypes.c_size_t, ctypes.c_uint32,
                                      ctypes.c_int, ctypes.c_uint64, ctypes.c_uint64,
                                      ctypes.c_void_p, ctypes.c_void_p]
        _cuda = L
    tb = torch.from_numpy(tables(seed)).to(t.device)
    s = stream if stream is not None else torch.cuda.current_stream(t.device)
    st = _cuda.syn_fill_device(ctypes.c_void_p(t.data_ptr()), t.numel(), chunk_size, cls, seed,
                               first_chunk, ctypes.c_void_p(tb.data_ptr()),
                               ctypes.c_void_p(s.cuda_stream))
    if st != 0:
        raise RuntimeError(f"syn_fill_device failed ({st})")
    s.synchronize()  # keep tb alive until the kernel has read it
    return t
