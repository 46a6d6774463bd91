"""CPU oracle -- TEST INFRASTRUCTURE ONLY.

ctypes wrapper over ``oracle/liblzr_ref.so`` (built from ``oracle/lzr_ref.c``,
plain serial greedy LZ77 over independent chunks; see that file for the paper
citations and DESIGN.md for the readings R1..R14).

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s CPU-baseline legs
(``cpu_baseline`` and ``--impl reference``) may import this package.  The
product path (``paper_conf_pact_map17_b200``) never imports it and shares no
code with it.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "liblzr_ref.so")
DEDUP_LIB_PATH = os.path.join(_HERE, "liblzr_dedup_ref.so")

OK = 0
ERR_INVALID_ARG = -1
ERR_UNSUPPORTED = -2
ERR_CAPACITY = -3
ERR_CORRUPT = -5


class _Params(ctypes.Structure):
    _fields_ = [
        ("chunk_size", ctypes.c_uint32),
        ("window", ctypes.c_uint32),
        ("min_match", ctypes.c_uint32),
        ("max_match", ctypes.c_uint32),
        ("tie_break", ctypes.c_uint32),
        ("parse", ctypes.c_uint32),
    ]


@dataclass(frozen=True)
class Params:
    chunk_size: int = 4096
    window: int | None = None  # None -> == chunk_size
    min_match: int = 4
    max_match: int | None = None  # None -> min_match + 255
    tie_break: int = 0
    parse: int = 0  # 0 = greedy (R8), 1 = one-step lazy (R21)

    def c(self) -> _Params:
        w = self.chunk_size if self.window is None else self.window
        mm = self.min_match + 255 if self.max_match is None else self.max_match
        return _Params(self.chunk_size, w, self.min_match, mm, self.tie_break, self.parse)


_lib = None


def build(force: bool = False) -> str:
    """Compile the oracle with plain gcc (no CUDA, no shared code)."""
    src = os.path.join(_HERE, "lzr_ref.c")
    if force or not os.path.exists(LIB_PATH) or os.path.getmtime(LIB_PATH) < max(
        os.path.getmtime(src), os.path.getmtime(os.path.join(_HERE, "lzr_ref.h"))
    ):
        import subprocess

        subprocess.check_call(
            ["gcc", "-O2", "-std=c11", "-Wall", "-Wextra", "-fPIC", "-shared", "-pthread",
             "-o", LIB_PATH + ".tmp", src]
        )
        os.replace(LIB_PATH + ".tmp", LIB_PATH)
    dsrc = os.path.join(_HERE, "dedup_ref.c")
    if force or not os.path.exists(DEDUP_LIB_PATH) or os.path.getmtime(DEDUP_LIB_PATH) < os.path.getmtime(dsrc):
        import subprocess

        subprocess.check_call(
            ["gcc", "-O2", "-std=c11", "-Wall", "-Wextra", "-fPIC", "-shared", "-pthread",
             "-o", DEDUP_LIB_PATH + ".tmp", dsrc]
        )
        os.replace(DEDUP_LIB_PATH + ".tmp", DEDUP_LIB_PATH)
    return LIB_PATH


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(LIB_PATH)
        P = ctypes.POINTER(_Params)
        u8p = ctypes.c_void_p
        L.lzr_ref_validate.argtypes = [P]
        L.lzr_ref_num_chunks.argtypes = [ctypes.c_size_t, P]
        L.lzr_ref_num_chunks.restype = ctypes.c_size_t
        L.lzr_ref_best_match.argtypes = [u8p, ctypes.c_size_t, ctypes.c_size_t, P,
                                         ctypes.POINTER(ctypes.c_uint32),
                                         ctypes.POINTER(ctypes.c_uint32)]
        L.lzr_ref_parse_chunk.argtypes = [u8p, ctypes.c_size_t, P, u8p, u8p]
        L.lzr_ref_parse_chunk.restype = ctypes.c_size_t
        L.lzr_ref_compress_chunk.argtypes = [u8p, ctypes.c_size_t, P, u8p]
        L.lzr_ref_compress_chunk.restype = ctypes.c_size_t
        L.lzr_ref_decompress_chunk.argtypes = [u8p, ctypes.c_size_t, ctypes.c_size_t, P, u8p]
        L.lzr_ref_compress.argtypes = [u8p, ctypes.c_size_t, P, u8p, ctypes.c_size_t, u8p, u8p,
                                       ctypes.POINTER(ctypes.c_uint64), ctypes.c_int]
        L.lzr_ref_compress_sampled.argtypes = [u8p, ctypes.c_size_t, P, u8p, ctypes.c_size_t,
                                               u8p, u8p, ctypes.c_int]
        L.lzr_ref_decompress.argtypes = [u8p, u8p, u8p, ctypes.c_size_t, P, u8p,
                                         ctypes.POINTER(ctypes.c_int32)]
        _lib = L
    return _lib


def _ptr(a: np.ndarray):
    return ctypes.c_void_p(a.ctypes.data)


def _u8(x) -> np.ndarray:
    if isinstance(x, (bytes, bytearray)):
        x = np.frombuffer(bytes(x), dtype=np.uint8)
    a = np.ascontiguousarray(x, dtype=np.uint8)
    return a


def validate(p: Params) -> int:
    return lib().lzr_ref_validate(ctypes.byref(p.c()))


def num_chunks(n: int, p: Params) -> int:
    return lib().lzr_ref_num_chunks(n, ctypes.byref(p.c()))


def best_match(x, p_pos: int, p: Params) -> tuple[int, int]:
    a = _u8(x)
    ln, dd = ctypes.c_uint32(), ctypes.c_uint32()
    lib().lzr_ref_best_match(_ptr(a), a.size, p_pos, ctypes.byref(p.c()), ctypes.byref(ln),
                             ctypes.byref(dd))
    return ln.value, dd.value


def parse_chunk(x, p: Params) -> list[tuple[int, int]]:
    """Greedy tokens of one chunk as (length, dist); dist 0 = literal."""
    a = _u8(x)
    n = max(1, a.size)
    lens = np.zeros(n, np.uint32)
    dists = np.zeros(n, np.uint32)
    T = lib().lzr_ref_parse_chunk(_ptr(a), a.size, ctypes.byref(p.c()), _ptr(lens), _ptr(dists))
    return [(int(lens[t]), int(dists[t])) for t in range(T)]


def compress_chunk(x, p: Params) -> bytes:
    a = _u8(x)
    out = np.zeros(max(1, a.size), np.uint8)
    S = lib().lzr_ref_compress_chunk(_ptr(a), a.size, ctypes.byref(p.c()), _ptr(out))
    return out[:S].tobytes()


def decompress_chunk(s, n: int, p: Params) -> tuple[int, bytes]:
    a = _u8(s)
    out = np.zeros(max(1, n), np.uint8)
    st = lib().lzr_ref_decompress_chunk(_ptr(a), a.size, n, ctypes.byref(p.c()), _ptr(out))
    return st, out[:n].tobytes()


def compress(x, p: Params, n_threads: int | None = None):
    """Whole stream -> (out bytes as np.uint8, sizes u32[N], offsets u64[N], total)."""
    a = _u8(x)
    if n_threads is None:
        n_threads = len(os.sched_getaffinity(0))
    N = num_chunks(a.size, p)
    out = np.zeros(max(1, a.size), np.uint8)
    sizes = np.zeros(max(1, N), np.uint32)
    offs = np.zeros(max(1, N), np.uint64)
    tot = ctypes.c_uint64()
    st = lib().lzr_ref_compress(_ptr(a), a.size, ctypes.byref(p.c()), _ptr(out), out.size,
                                _ptr(sizes), _ptr(offs), ctypes.byref(tot), n_threads)
    if st != OK:
        raise ValueError(f"lzr_ref_compress status {st}")
    return out[: tot.value], sizes[:N], offs[:N], tot.value


def compress_sampled(x, p: Params, idx, n_threads: int | None = None):
    """Compress only chunks idx -> list of per-chunk byte strings."""
    a = _u8(x)
    if n_threads is None:
        n_threads = len(os.sched_getaffinity(0))
    ix = np.ascontiguousarray(idx, dtype=np.uint64)
    out = np.zeros(max(1, ix.size * p.chunk_size), np.uint8)
    sizes = np.zeros(max(1, ix.size), np.uint32)
    st = lib().lzr_ref_compress_sampled(_ptr(a), a.size, ctypes.byref(p.c()), _ptr(ix), ix.size,
                                        _ptr(out), _ptr(sizes), n_threads)
    if st != OK:
        raise ValueError(f"lzr_ref_compress_sampled status {st}")
    C = p.chunk_size
    return [out[k * C: k * C + int(sizes[k])].tobytes() for k in range(ix.size)], sizes[: ix.size]


def decompress(comp, sizes, offsets, n: int, p: Params) -> tuple[int, int, np.ndarray]:
    """-> (status, first_bad (1+index or 0), output)."""
    c = _u8(comp)
    if c.size == 0:
        c = np.zeros(1, np.uint8)
    s = np.ascontiguousarray(sizes, dtype=np.uint32)
    o = np.ascontiguousarray(offsets, dtype=np.uint64)
    out = np.zeros(max(1, n), np.uint8)
    bad = ctypes.c_int32()
    st = lib().lzr_ref_decompress(_ptr(c), _ptr(s), _ptr(o), n, ctypes.byref(p.c()), _ptr(out),
                                  ctypes.byref(bad))
    return st, bad.value, out[:n]


# ---- dedup (oracle/dedup_ref.c) -------------
_dlib = None


def dlib():
    global _dlib
    if _dlib is None:
        build()
        L = ctypes.CDLL(DEDUP_LIB_PATH)
        L.dedup_ref_sha1.argtypes = [ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p]
        L.dedup_ref_fingerprints.argtypes = [ctypes.c_void_p, ctypes.c_size_t, ctypes.c_size_t,
                                             ctypes.c_void_p, ctypes.c_int]
        _dlib = L
    return _dlib


def sha1(x) -> bytes:
    """SHA-1 digest of a byte string (plain C, FIPS 180-4)."""
    a = _u8(x)
    buf = a if a.size else np.zeros(1, np.uint8)
    out = np.zeros(20, np.uint8)
    dlib().dedup_ref_sha1(_ptr(buf), a.size, _ptr(out))
    return out.tobytes()


def fingerprints(x, chunk_size: int, n_threads: int | None = None) -> np.ndarray:
    """fp[i] = SHA-1 of chunk i -> uint8[N, 20].  P:12 §2 "Hashing is the process of
    calculating the hash value of each chunk"; §3.1(1) "SHA1, 20 bytes"."""
    a = _u8(x)
    if n_threads is None:
        n_threads = len(os.sched_getaffinity(0))
    N = (a.size + chunk_size - 1) // chunk_size
    fp = np.zeros((max(1, N), 20), np.uint8)
    buf = a if a.size else np.zeros(1, np.uint8)
    st = dlib().dedup_ref_fingerprints(_ptr(buf), a.size, chunk_size, _ptr(fp), n_threads)
    if st != 0:
        raise ValueError(f"dedup_ref_fingerprints status {st}")
    return fp[:N]


def dedup_index(fps: np.ndarray, first_chunk: int = 0, seen: dict | None = None):
    """Indexing step (§2 "Indexing is the process of comparing the hash value of
    each chunk with the hash values of already stored chunks to determine whether it
    is a duplicate"; §3.1(2) "the result of whether an index is hit or not
    includes an index number and a hit/miss information pair").

    Chunks are indexed in stream order; the index number of chunk i (global index
    first_chunk + i) is the global index of the first chunk with the same
    fingerprint (itself when it is new: a miss).  ``seen`` carries the index
    across batches (fingerprint bytes -> first global index).
    Returns (index uint64[N], hit uint8[N], seen)."""
    if seen is None:
        seen = {}
    N = len(fps)
    index = np.zeros(N, np.uint64)
    hit = np.zeros(N, np.uint8)
    for i in range(N):
        key = bytes(fps[i])
        g = first_chunk + i
        if key in seen:
            index[i] = seen[key]
            hit[i] = 1
        else:
            seen[key] = g
            index[i] = g
    return index, hit, seen
