"""B200-native chunked LZ compression (Ma & Park, PaCT 2017 -- the GPU side of
inline compression of fixed-size write chunks).

Thin Python binding over the C ABI of ``liblzr.so`` (``include/lzr.h``):
argument marshalling only.  Every step of the path (staging, match search,
greedy token selection, encoding, scan, compaction, decoding) runs in the
sm_100a kernels of ``csrc/``.  PyTorch is used for device memory and streams.
There is no CPU fallback: importing this package fails loudly when the CUDA
library has not been built, and the compute calls need a CUDA device.
"""
from __future__ import annotations

import contextlib
import ctypes
import os
from dataclasses import dataclass

__all__ = [
    "Params", "LzrError", "lib", "num_chunks", "compress_bound", "compress_workspace_bytes",
    "compress", "compress_encode", "compress_compact", "scan_sizes", "decompress",
    "compress_host", "decompress_host", "validate_params", "status_str", "last_launch_count",
    "fingerprint", "DedupIndex", "gather_chunks", "dedup_compress", "owner_counts", "route",
    "unroute",
]

_PKG = os.path.dirname(os.path.abspath(__file__))
# LZR_LIBRARY may point at an instrumented build of the same sources (profiling)
LIB_PATH = os.environ.get("LZR_LIBRARY") or os.path.join(_PKG, "liblzr.so")

OK, ERR_INVALID_ARG, ERR_UNSUPPORTED, ERR_CAPACITY, ERR_CUDA, ERR_CORRUPT = 0, -1, -2, -3, -4, -5
PARSE_GREEDY, PARSE_LAZY = 0, 1  # lzr_params.parse (include/lzr.h; R8, R21)

EXPORTED_SYMBOLS = [
    "lzr_validate_params", "lzr_num_chunks", "lzr_compress_bound", "lzr_compress_workspace_bytes",
    "lzr_compress_chunks", "lzr_compress_encode", "lzr_compress_compact",
    "lzr_scan_workspace_bytes", "lzr_scan_sizes", "lzr_decompress_workspace_bytes", "lzr_decompress_chunks",
    "lzr_compress_host_scratch_bytes", "lzr_compress_host", "lzr_status_str",
    "lzr_last_launch_count", "lzr_fingerprint_chunks", "lzr_dedup_table_bytes", "lzr_dedup_index",
    "lzr_gather_chunks", "lzr_dedup_index_gidx", "lzr_dedup_owner_counts", "lzr_dedup_route",
    "lzr_dedup_unroute", "lzr_decompress_host_scratch_bytes", "lzr_decompress_host",
]


class LzrError(RuntimeError):
    def __init__(self, status: int, what: str):
        super().__init__(f"{what}: {status_str(status)} ({status})")
        self.status = status


class _CParams(ctypes.Structure):
    _fields_ = [("chunk_size", ctypes.c_uint32), ("window", ctypes.c_uint32),
                ("min_match", ctypes.c_uint32), ("max_match", ctypes.c_uint32),
                ("tie_break", ctypes.c_uint32), ("parse", ctypes.c_uint32)]


@dataclass(frozen=True)
class Params:
    """lzr_params.  Defaults: C = W = 4096, m = 4, M = m + 255 (R1-R7)."""
    chunk_size: int = 4096
    window: int | None = None
    min_match: int = 4
    max_match: int | None = None
    tie_break: int = 0
    parse: int = 0  # PARSE_GREEDY (R8) or PARSE_LAZY (R21)

    def c(self) -> _CParams:
        w = self.chunk_size if self.window is None else self.window
        mm = self.min_match + 255 if self.max_match is None else self.max_match
        return _CParams(self.chunk_size, w, self.min_match, mm, self.tie_break, self.parse)


_lib = None


def lib():
    """Load liblzr.so.  Raises if it has not been built (no fallback path)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(
                f"{LIB_PATH} is missing: build it with `python -c 'import __graft_entry__ as g; "
                "g.build()'` (nvcc, sm_100a).  There is no CPU fallback.")
        L = ctypes.CDLL(LIB_PATH)
        P = ctypes.POINTER(_CParams)
        vp, sz, u64 = ctypes.c_void_p, ctypes.c_size_t, ctypes.c_uint64
        L.lzr_validate_params.argtypes = [P]
        L.lzr_num_chunks.argtypes = [sz, P]
        L.lzr_num_chunks.restype = sz
        L.lzr_compress_bound.argtypes = [sz, P]
        L.lzr_compress_bound.restype = sz
        L.lzr_compress_workspace_bytes.argtypes = [sz, P]
        L.lzr_compress_workspace_bytes.restype = sz
        L.lzr_compress_chunks.argtypes = [vp, sz, P, vp, sz, vp, vp, vp, vp, sz, vp]
        L.lzr_compress_encode.argtypes = [vp, sz, P, vp, vp, sz, vp]
        L.lzr_compress_compact.argtypes = [vp, sz, P, vp, sz, vp, vp, vp, vp, sz, vp]
        L.lzr_scan_workspace_bytes.argtypes = [sz]
        L.lzr_scan_workspace_bytes.restype = sz
        L.lzr_scan_sizes.argtypes = [vp, sz, u64, vp, vp, vp, sz, vp]
        L.lzr_decompress_workspace_bytes.argtypes = [sz, P]
        L.lzr_decompress_workspace_bytes.restype = sz
        L.lzr_decompress_chunks.argtypes = [vp, vp, vp, sz, P, vp, vp, vp, sz, vp]
        L.lzr_compress_host_scratch_bytes.argtypes = [sz, P]
        L.lzr_compress_host_scratch_bytes.restype = sz
        L.lzr_compress_host.argtypes = [vp, sz, P, vp, sz, vp, vp, vp, sz, vp, sz]
        L.lzr_decompress_host_scratch_bytes.argtypes = [sz, P]
        L.lzr_decompress_host_scratch_bytes.restype = sz
        L.lzr_decompress_host.argtypes = [vp, vp, vp, sz, P, vp, vp, sz, vp, sz]
        L.lzr_status_str.argtypes = [ctypes.c_int]
        L.lzr_status_str.restype = ctypes.c_char_p
        L.lzr_last_launch_count.argtypes = []
        L.lzr_fingerprint_chunks.argtypes = [vp, sz, ctypes.c_uint32, vp, vp]
        L.lzr_dedup_table_bytes.argtypes = [ctypes.c_uint32, ctypes.c_uint32]
        L.lzr_dedup_table_bytes.restype = sz
        L.lzr_dedup_index.argtypes = [vp, sz, u64, vp, ctypes.c_uint32, ctypes.c_uint32, vp, vp, vp,
                                      vp]
        L.lzr_gather_chunks.argtypes = [vp, sz, ctypes.c_uint32, vp, vp, vp, vp]
        L.lzr_dedup_index_gidx.argtypes = [vp, sz, vp, vp, ctypes.c_uint32, ctypes.c_uint32, vp, vp,
                                           vp, vp]
        L.lzr_dedup_owner_counts.argtypes = [vp, sz, ctypes.c_uint32, vp, vp]
        L.lzr_dedup_route.argtypes = [vp, sz, u64, ctypes.c_uint32, vp, vp, vp, vp, vp, vp]
        L.lzr_dedup_unroute.argtypes = [vp, vp, sz, u64, vp, vp, vp]
        _lib = L
    return _lib


def status_str(st: int) -> str:
    return lib().lzr_status_str(st).decode()


def _check(st: int, what: str):
    if st != OK:
        raise LzrError(st, what)


def validate_params(p: Params) -> int:
    return lib().lzr_validate_params(ctypes.byref(p.c()))


def num_chunks(n: int, p: Params) -> int:
    return lib().lzr_num_chunks(n, ctypes.byref(p.c()))


def compress_bound(n: int, p: Params) -> int:
    return lib().lzr_compress_bound(n, ctypes.byref(p.c()))


def compress_workspace_bytes(n: int, p: Params) -> int:
    return lib().lzr_compress_workspace_bytes(n, ctypes.byref(p.c()))


def last_launch_count() -> int:
    return lib().lzr_last_launch_count()


def _ptr(t):
    return ctypes.c_void_p(t.data_ptr() if t is not None and t.numel() else 0)


def _stream(stream, device):
    import torch

    s = stream if stream is not None else torch.cuda.current_stream(device)
    return ctypes.c_void_p(s.cuda_stream)


@contextlib.contextmanager
def _on(device, stream=None):
    """Run liblzr calls with `device` current (the C ABI launches on the
    current device, include/lzr.h) and, when a stream is given, with it as
    torch's current stream, so that buffers allocated here belong to it and
    host reads (.item()) synchronise with the work launched on it."""
    import torch

    with contextlib.ExitStack() as es:
        dev = torch.device(device) if device is not None else None
        if dev is not None and dev.type == "cuda":
            es.enter_context(torch.cuda.device(dev))
        if stream is not None:
            es.enter_context(torch.cuda.stream(stream))
        yield


def _same_device(*ts):
    devs = {t.device for t in ts if t is not None}
    if len(devs) > 1:
        raise ValueError(f"tensors on different devices: {sorted(map(str, devs))}")


def _require_cuda_u8(t, name):
    import torch

    if not (isinstance(t, torch.Tensor) and t.is_cuda and t.dtype == torch.uint8 and t.is_contiguous()):
        raise TypeError(f"{name} must be a contiguous uint8 CUDA tensor")


class Workspace:
    """Reusable device buffers for repeated compress() calls of one size."""

    def __init__(self, n: int, p: Params, device=None):
        import torch

        self.n, self.p = n, p
        dev = torch.device(device) if device is not None else torch.device("cuda", torch.cuda.current_device())
        N = num_chunks(n, p)
        with _on(dev):  # the workspace size depends on the device's SM count
            self.out = torch.empty(max(1, compress_bound(n, p)), dtype=torch.uint8, device=dev)
            self.sizes = torch.empty(max(1, N), dtype=torch.int32, device=dev)
            self.offsets = torch.empty(max(1, N), dtype=torch.int64, device=dev)
            self.total = torch.zeros(1, dtype=torch.int64, device=dev)
            self.ws = torch.empty(max(256, compress_workspace_bytes(n, p)), dtype=torch.uint8,
                                  device=dev)
        self.device = dev
        self.N = N


def compress(t, p: Params = Params(), ws: Workspace | None = None, stream=None):
    """Compress a uint8 CUDA tensor chunk by chunk.

    Returns (out, sizes, offsets, total): ``out`` holds ``capacity = n`` bytes of
    which the first ``total`` are the compacted chunk streams; ``sizes`` int32
    (bit pattern of the ABI's uint32), ``offsets`` int64, ``total`` int64[1] --
    all device tensors; nothing is synchronised.
    """
    _require_cuda_u8(t, "input")
    n = t.numel()
    with _on(t.device, stream):
        if ws is None or ws.n != n or ws.p != p:
            ws = Workspace(n, p, t.device)
        _same_device(t, ws.ws)
        st = lib().lzr_compress_chunks(
            _ptr(t), n, ctypes.byref(p.c()), _ptr(ws.out), ws.out.numel(), _ptr(ws.sizes),
            _ptr(ws.offsets), _ptr(ws.total), _ptr(ws.ws), ws.ws.numel(), _stream(stream, t.device))
    _check(st, "lzr_compress_chunks")
    N = ws.N
    return ws.out, ws.sizes[:N], ws.offsets[:N], ws.total


def compress_encode(t, p: Params, ws: Workspace, stream=None):
    """Launch only the encode stage (bench timing): sizes in ws.sizes."""
    _same_device(t, ws.ws)
    with _on(t.device, stream):
        st = lib().lzr_compress_encode(_ptr(t), t.numel(), ctypes.byref(p.c()), _ptr(ws.sizes),
                                       _ptr(ws.ws), ws.ws.numel(), _stream(stream, t.device))
    _check(st, "lzr_compress_encode")


def compress_compact(t, p: Params, ws: Workspace, stream=None):
    """Launch only the scan + compaction stage (after compress_encode)."""
    _same_device(t, ws.ws)
    with _on(t.device, stream):
        st = lib().lzr_compress_compact(
            _ptr(t), t.numel(), ctypes.byref(p.c()), _ptr(ws.out), ws.out.numel(), _ptr(ws.sizes),
            _ptr(ws.offsets), _ptr(ws.total), _ptr(ws.ws), ws.ws.numel(), _stream(stream, t.device))
    _check(st, "lzr_compress_compact")


def scan_sizes(sizes, base: int = 0, offsets=None, total=None, ws=None, stream=None):
    """Exclusive prefix sum (+ base) of int32/uint32 sizes on the device."""
    import torch

    n = sizes.numel()
    with _on(sizes.device, stream):
        if offsets is None:
            offsets = torch.empty(max(1, n), dtype=torch.int64, device=sizes.device)
        if total is None:
            total = torch.zeros(1, dtype=torch.int64, device=sizes.device)
        wsb = lib().lzr_scan_workspace_bytes(n)
        if ws is None or ws.numel() < wsb:
            ws = torch.empty(max(256, wsb), dtype=torch.uint8, device=sizes.device)
        _same_device(sizes, offsets, total, ws)
        st = lib().lzr_scan_sizes(_ptr(sizes), n, base, _ptr(offsets), _ptr(total), _ptr(ws),
                                  ws.numel(), _stream(stream, sizes.device))
    _check(st, "lzr_scan_sizes")
    return offsets[:n], total


def decompress(comp, sizes, offsets, n: int, p: Params = Params(), out=None, error=None,
               stream=None, workspace=None, schedule: bool = True):
    """Decode chunk streams back into n bytes.  Returns (out, error) where
    error is an int32[1] device tensor: 0 or 1 + index of the first corrupt chunk.
    schedule: decode the chunks costliest first (needs a workspace of
    lzr_decompress_workspace_bytes; allocated here when not given); the
    output is the same either way."""
    import torch

    dev = comp.device
    with _on(dev, stream):
        if out is None:
            out = torch.empty(max(1, n), dtype=torch.uint8, device=dev)
        if error is None:
            error = torch.zeros(1, dtype=torch.int32, device=dev)
        ws_bytes = 0
        if schedule:
            ws_bytes = lib().lzr_decompress_workspace_bytes(n, ctypes.byref(p.c()))
            if workspace is None:
                workspace = torch.empty(max(1, ws_bytes), dtype=torch.uint8, device=dev)
            _same_device(comp, workspace)
            ws_bytes = workspace.numel()
        _same_device(comp, sizes, offsets, out, error)
        st = lib().lzr_decompress_chunks(_ptr(comp), _ptr(sizes), _ptr(offsets), n,
                                         ctypes.byref(p.c()), _ptr(out), _ptr(error),
                                         _ptr(workspace) if schedule else None, ws_bytes,
                                         _stream(stream, dev))
    _check(st, "lzr_decompress_chunks")
    return out[:n], error


def compress_host(h_in, p: Params = Params(), batch_bytes: int = 16 << 20, scratch=None,
                  h_out=None, h_sizes=None, h_offsets=None):
    """End-to-end compression of a host (preferably pinned) uint8 tensor through
    the C ABI's host-buffer pipeline (H2D, kernels, D2H inside; 16 MiB batches
    by default, 0 = one batch).  Synchronous.
    Returns (h_out, h_sizes, h_offsets, total) on the host."""
    import torch

    n = h_in.numel()
    N = num_chunks(n, p)
    batch_bytes = -(-batch_bytes // p.chunk_size) * p.chunk_size
    if batch_bytes == 0 or batch_bytes > n:
        batch_bytes = max(p.chunk_size, -(-n // p.chunk_size) * p.chunk_size)
    need = lib().lzr_compress_host_scratch_bytes(batch_bytes, ctypes.byref(p.c()))
    if scratch is None or scratch.numel() < need:
        scratch = torch.empty(max(256, need), dtype=torch.uint8, device="cuda")
    if h_out is None:
        h_out = torch.empty(max(1, n), dtype=torch.uint8, pin_memory=True)
    if h_sizes is None:
        h_sizes = torch.empty(max(1, N), dtype=torch.int32, pin_memory=True)
    if h_offsets is None:
        h_offsets = torch.empty(max(1, N), dtype=torch.int64, pin_memory=True)
    tot = ctypes.c_uint64()
    st = lib().lzr_compress_host(
        ctypes.c_void_p(h_in.data_ptr()), n, ctypes.byref(p.c()), ctypes.c_void_p(h_out.data_ptr()),
        h_out.numel(), ctypes.c_void_p(h_sizes.data_ptr()), ctypes.c_void_p(h_offsets.data_ptr()),
        ctypes.byref(tot), batch_bytes, _ptr(scratch), scratch.numel())
    _check(st, "lzr_compress_host")
    return h_out, h_sizes[:N], h_offsets[:N], tot.value


def decompress_host(h_comp, h_sizes, h_offsets, n: int, p: Params = Params(), batch_bytes: int = 16 << 20,
                    scratch=None, h_out=None):
    """End-to-end decompression of host (preferably pinned) buffers through the
    C ABI's host pipeline (H2D of each batch's streams, decode, D2H inside).
    Synchronous.  Returns (h_out, error): error 0 or 1 + index of the first
    corrupt chunk."""
    import torch

    batch_bytes = -(-batch_bytes // p.chunk_size) * p.chunk_size
    if batch_bytes == 0 or batch_bytes > n:
        batch_bytes = max(p.chunk_size, -(-n // p.chunk_size) * p.chunk_size)
    need = lib().lzr_decompress_host_scratch_bytes(batch_bytes, ctypes.byref(p.c()))
    if scratch is None or scratch.numel() < need:
        scratch = torch.empty(max(256, need), dtype=torch.uint8, device="cuda")
    if h_out is None:
        h_out = torch.empty(max(1, n), dtype=torch.uint8, pin_memory=True)
    err = ctypes.c_int32()
    st = lib().lzr_decompress_host(
        ctypes.c_void_p(h_comp.data_ptr()), ctypes.c_void_p(h_sizes.data_ptr()),
        ctypes.c_void_p(h_offsets.data_ptr()), n, ctypes.byref(p.c()), ctypes.c_void_p(h_out.data_ptr()),
        ctypes.byref(err), batch_bytes, _ptr(scratch), scratch.numel())
    _check(st, "lzr_decompress_host")
    return h_out[:n], err.value


# ---- dedup upstream of compression (include/lzr.h) ---------------
def fingerprint(t, chunk_size: int = 4096, out=None, stream=None):
    """SHA-1 of every chunk of a uint8 CUDA tensor -> uint8[N, 20] CUDA tensor."""
    import torch

    _require_cuda_u8(t, "input")
    n = t.numel()
    N = -(-n // chunk_size)
    with _on(t.device, stream):
        if out is None:
            out = torch.empty((max(1, N), 20), dtype=torch.uint8, device=t.device)
        _same_device(t, out)
        st = lib().lzr_fingerprint_chunks(_ptr(t), n, chunk_size, _ptr(out), _stream(stream, t.device))
    _check(st, "lzr_fingerprint_chunks")
    return out[:N]


class DedupIndex:
    """Bin-partitioned fingerprint index kept on the device across batches
    (n_bins bins x bin_slots entries; zero-filled = empty)."""

    def __init__(self, n_bins: int, bin_slots: int, device=None):
        import torch

        self.n_bins, self.bin_slots = n_bins, bin_slots
        dev = torch.device(device) if device is not None else torch.device("cuda", torch.cuda.current_device())
        nb = lib().lzr_dedup_table_bytes(n_bins, bin_slots)
        with _on(dev):
            self.table = torch.zeros(max(256, nb), dtype=torch.uint8, device=dev)
            self.overflow = torch.zeros(1, dtype=torch.int32, device=dev)

    @classmethod
    def for_chunks(cls, n_chunks: int, device=None, bin_slots: int = 64):
        """Sized for n_chunks fingerprints at <= 50% load."""
        n_bins = max(1, -(-2 * max(1, n_chunks) // bin_slots))
        return cls(n_bins, bin_slots, device)

    def reset(self):
        self.table.zero_()
        self.overflow.zero_()

    def index(self, fp, first_chunk: int = 0, index=None, unique=None, stream=None):
        """-> (index int64[N]: first global index with the same fingerprint,
        unique int32[N]: 1 on a miss).  Nothing is synchronised."""
        import torch

        N = fp.shape[0]
        dev = fp.device
        with _on(dev, stream):
            if index is None:
                index = torch.empty(max(1, N), dtype=torch.int64, device=dev)
            if unique is None:
                unique = torch.empty(max(1, N), dtype=torch.int32, device=dev)
            _same_device(fp, self.table, index, unique)
            st = lib().lzr_dedup_index(_ptr(fp), N, first_chunk, _ptr(self.table), self.n_bins,
                                       self.bin_slots, _ptr(index), _ptr(unique), _ptr(self.overflow),
                                       _stream(stream, dev))
        _check(st, "lzr_dedup_index")
        return index[:N], unique[:N]

    def index_gidx(self, fp, gidx, stream=None):
        """Owner side of the multi-GPU index: record i's global index is gidx[i]."""
        import torch

        N = fp.shape[0]
        dev = fp.device
        with _on(dev, stream):
            index = torch.empty(max(1, N), dtype=torch.int64, device=dev)
            unique = torch.empty(max(1, N), dtype=torch.int32, device=dev)
            _same_device(fp, gidx, self.table)
            st = lib().lzr_dedup_index_gidx(_ptr(fp), N, _ptr(gidx), _ptr(self.table), self.n_bins,
                                            self.bin_slots, _ptr(index), _ptr(unique),
                                            _ptr(self.overflow), _stream(stream, dev))
        _check(st, "lzr_dedup_index_gidx")
        return index[:N], unique[:N]


def owner_counts(fp, n_owners: int, counts=None, stream=None):
    """Per-owner fingerprint counts (int32[n_owners], zeroed here) for the
    multi-GPU index (include/lzr.h lzr_dedup_owner_counts)."""
    import torch

    with _on(fp.device, stream):
        if counts is None:
            counts = torch.zeros(n_owners, dtype=torch.int32, device=fp.device)
        else:
            counts.zero_()
        _same_device(fp, counts)
        st = lib().lzr_dedup_owner_counts(_ptr(fp), fp.shape[0], n_owners, _ptr(counts),
                                          _stream(stream, fp.device))
    _check(st, "lzr_dedup_owner_counts")
    return counts


def route(fp, first_chunk: int, n_owners: int, base, stream=None):
    """Records (fingerprint, global index) grouped by owner in send order ->
    (send_fp uint8[N,20], send_gidx int64[N], slot int32[N])."""
    import torch

    N = fp.shape[0]
    dev = fp.device
    with _on(dev, stream):
        cursor = torch.zeros(n_owners, dtype=torch.int32, device=dev)
        send_fp = torch.empty((max(1, N), 20), dtype=torch.uint8, device=dev)
        send_gidx = torch.empty(max(1, N), dtype=torch.int64, device=dev)
        slot = torch.empty(max(1, N), dtype=torch.int32, device=dev)
        _same_device(fp, base)
        st = lib().lzr_dedup_route(_ptr(fp), N, first_chunk, n_owners, _ptr(base), _ptr(cursor),
                                   _ptr(send_fp), _ptr(send_gidx), _ptr(slot), _stream(stream, dev))
    _check(st, "lzr_dedup_route")
    return send_fp[:N], send_gidx[:N], slot[:N]


def unroute(back, slot, first_chunk: int, stream=None):
    """Owners' index numbers (send order) -> (index int64[N], unique int32[N]) in chunk order."""
    import torch

    N = slot.shape[0]
    dev = slot.device
    with _on(dev, stream):
        index = torch.empty(max(1, N), dtype=torch.int64, device=dev)
        unique = torch.empty(max(1, N), dtype=torch.int32, device=dev)
        _same_device(back, slot)
        st = lib().lzr_dedup_unroute(_ptr(back), _ptr(slot), N, first_chunk, _ptr(index), _ptr(unique),
                                     _stream(stream, dev))
    _check(st, "lzr_dedup_unroute")
    return index[:N], unique[:N]


def gather_chunks(t, chunk_size: int, unique, rank, out, stream=None):
    """Copy the unique chunks of t to out in stream order (out + rank[i] * C)."""
    _same_device(t, unique, rank, out)
    with _on(t.device, stream):
        st = lib().lzr_gather_chunks(_ptr(t), t.numel(), chunk_size, _ptr(unique), _ptr(rank),
                                     _ptr(out), _stream(stream, t.device))
    _check(st, "lzr_gather_chunks")
    return out


def dedup_compress(t, p: Params = Params(), index: DedupIndex | None = None, first_chunk: int = 0,
                   ws: Workspace | None = None, stream=None):
    """Dedup before compression (§3.3): fingerprint every chunk, index the
    fingerprints, gather the unique chunks, compress them.  Synchronises once to
    size the unique buffer.  Returns a dict with fp, index, unique, rank,
    n_unique, the gathered unique bytes and compress()'s (out, sizes, offsets,
    total) over them.

    Trust assumption (§3.1(1): the index keys are SHA-1 fingerprints): two
    chunks with equal SHA-1 are treated as duplicates without a byte compare,
    as in the paper; a deliberately constructed SHA-1 collision would drop the
    second chunk's content (R17)."""
    import torch

    C = p.chunk_size
    # everything below runs on `stream` (and t's device), so the host reads of
    # the unique count wait for the kernels that produce it
    with _on(t.device, stream):
        if index is None:
            index = DedupIndex.for_chunks(-(-t.numel() // C), t.device)
        fp = fingerprint(t, C, stream=stream)
        idx, uniq = index.index(fp, first_chunk, stream=stream)
        rank, n_uniq_t = scan_sizes(uniq, stream=stream)
        n = t.numel()
        N = fp.shape[0]
        nu = int(n_uniq_t.item())
        last_unique = N > 0 and bool(uniq[N - 1].item())
        ubytes = nu * C
        if last_unique and n % C:
            ubytes -= C - n % C  # the short tail chunk is the last unique one
        ubuf = torch.empty(max(1, ubytes), dtype=torch.uint8, device=t.device)
        gather_chunks(t, C, uniq, rank, ubuf, stream=stream)
        u = ubuf[:ubytes]
        out, sizes, offs, total = compress(u, p, ws=ws, stream=stream)
    return {"fp": fp, "index": idx, "unique": uniq, "rank": rank, "n_unique": nu, "unique_bytes": u,
            "out": out, "sizes": sizes, "offsets": offs, "total": total}
