"""Fast exact CPU compressor -- the paper's CPU arm, TEST INFRASTRUCTURE AND
CPU BASELINE (``cpuref/lzr_fast.c``).

The same result as the plain oracle (``oracle/``), found with hash chains and
a run-aware search instead of an exhaustive scan, multi-threaded per chunk
(§3.2(1)).  Pinned to the oracle by ``tests/test_cpuref.py``.  Used for
whole-stream GPU parity at multi-GiB sizes, as the CPU arm of the paper's
GPU-usage decision (§3.2(3)) in ``bench.py``, and injected by bench.py /
the tests as the CPU side of the integration-option selection
(``paper_conf_pact_map17_b200.integration``, §4(3)).  Only ``tests/``,
``bench.py`` and ``tools/`` import it; the product package never does.
``dedup`` is the CPU dedup arm (hashlib SHA-1 + a first-occurrence dict, R17/R18).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "liblzr_fast.so")


class _Params(ctypes.Structure):
    _fields_ = [(f, ctypes.c_uint32) for f in
                ("chunk_size", "window", "min_match", "max_match", "tie_break", "parse")]


@dataclass(frozen=True)
class Params:
    chunk_size: int = 4096
    window: int | None = None
    min_match: int = 4
    max_match: int | None = None
    tie_break: int = 0
    parse: int = 0

    def c(self) -> _Params:
        w = self.chunk_size if self.window is None else self.window
        mm = self.min_match + 255 if self.max_match is None else self.max_match
        return _Params(self.chunk_size, w, self.min_match, mm, self.tie_break, self.parse)


def build(force: bool = False) -> str:
    src = [os.path.join(_HERE, f) for f in ("lzr_fast.c", "lzr_fast.h")]
    if force or not os.path.exists(LIB_PATH) or os.path.getmtime(LIB_PATH) < max(map(os.path.getmtime, src)):
        subprocess.check_call(["gcc", "-O3", "-march=x86-64-v2", "-std=c11", "-Wall", "-Wextra", "-fPIC",
                               "-shared", "-pthread", "-o", LIB_PATH + ".tmp", src[0]])
        os.replace(LIB_PATH + ".tmp", LIB_PATH)
    return LIB_PATH


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(LIB_PATH)
        vp = ctypes.c_void_p
        L.lzr_fast_compress.argtypes = [vp, ctypes.c_size_t, ctypes.POINTER(_Params), vp, vp, vp, vp,
                                        vp, ctypes.c_int]
        L.lzr_fast_compress.restype = ctypes.c_int
        L.lzr_fast_validate.argtypes = [ctypes.POINTER(_Params)]
        _lib = L
    return _lib


def validate(p: Params) -> int:
    return lib().lzr_fast_validate(ctypes.byref(p.c()))


def _ptr(a: np.ndarray):
    return ctypes.c_void_p(a.ctypes.data)


def compress(x, p: Params, n_threads: int | None = None, slots: np.ndarray | None = None):
    """-> (out u8 view of length total, sizes u32[N], offsets u64[N], total); like oracle.compress.
    ``slots`` (>= len(x) bytes) is reused as the output buffer when given."""
    a = np.ascontiguousarray(np.frombuffer(x, np.uint8) if isinstance(x, (bytes, bytearray)) else x,
                             dtype=np.uint8).reshape(-1)
    if n_threads is None:
        n_threads = len(os.sched_getaffinity(0))
    N = (a.size + p.chunk_size - 1) // p.chunk_size
    buf = slots if slots is not None and slots.size >= a.size else np.empty(max(1, a.size), np.uint8)
    sizes = np.zeros(max(1, N), np.uint32)
    offs = np.zeros(max(1, N), np.uint64)
    tot = ctypes.c_uint64()
    st = lib().lzr_fast_compress(_ptr(a), a.size, ctypes.byref(p.c()), _ptr(buf), _ptr(buf),
                                 _ptr(sizes), _ptr(offs), ctypes.byref(tot), n_threads)
    if st != 0:
        raise ValueError(f"lzr_fast_compress status {st}")
    return buf[: tot.value], sizes[:N], offs[:N], tot.value


def dedup(x, chunk_size: int, n_threads: int | None = None):
    """CPU dedup arm: SHA-1 of every chunk (hashlib, threads; a short tail chunk
    hashes its own length, R17), then first-occurrence indexing in stream order
    (R18).  -> (index int64[N], unique int32[N])."""
    import hashlib
    from concurrent.futures import ThreadPoolExecutor

    a = np.ascontiguousarray(x, dtype=np.uint8).reshape(-1)
    C = chunk_size
    N = -(-a.size // C)
    mv = memoryview(a)
    if n_threads is None:
        n_threads = len(os.sched_getaffinity(0))
    step = max(1, -(-N // (4 * n_threads)))

    def part(lo):
        return [hashlib.sha1(mv[i * C: min(a.size, (i + 1) * C)]).digest() for i in range(lo, min(N, lo + step))]

    with ThreadPoolExecutor(n_threads) as ex:
        fps = [d for blk in ex.map(part, range(0, N, step)) for d in blk]
    first = {}
    index = np.empty(N, np.int64)
    for i, d in enumerate(fps):
        index[i] = first.setdefault(d, i)
    unique = (index == np.arange(N)).astype(np.int32)
    return index, unique
