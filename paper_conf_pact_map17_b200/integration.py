"""Integration-option selection by dummy I/O (PAPER.md
P:20 §4(3): "The first option is to use the GPU in two data reduction
operations ... only one ... both ... do not use the GPU" -- the options are
"compared using dummy I/O to determine the best fit for throughput"; P:16
§3.2(3) "we compare the compression performance of the CPU and the GPU to
determine when to use the GPU").

The integrated write path is dedup before compression (§3.3): every
chunk of a host-resident write stream is fingerprinted and indexed, and only
the unique chunks are compressed.  A *placement* says where each of the two
reductions runs:

  gpu_both                 GPU dedup (SHA-1, bin index, gather) + GPU compression
  gpu_dedup_cpu_compress   GPU dedup, the unique chunks compressed on the CPU
  cpu_dedup_gpu_compress   CPU dedup, the unique chunks compressed on the GPU
  cpu_both                 no GPU
  gpu_dedup_split          GPU dedup, the unique chunks split between the GPU
                           and the CPU compressor (fraction f on the CPU, f from
                           the two measured compression rates), run concurrently

Every placement computes the same result (index numbers, unique flags and
the compressed bytes of the unique stream, R17/R18 and R1-R9), so the choice
is throughput only.  ``Integrated.calibrate`` runs a dummy stream through each
placement, end to end from host memory (the stream arrives by I/O; H2D/D2H are
inside the GPU placements' times) and picks the fastest.

This package has no CPU implementation of the method: the CPU arm (compressor
and dedup) is injected by the caller as a ``CpuArm`` (bench.py and the tests
pass the fast exact CPU compressor ``cpuref`` and a hashlib-based dedup).
``compress()`` / ``decompress()`` never route through it.
"""
from __future__ import annotations

import threading
import time
from dataclasses import dataclass
from typing import Callable

import numpy as np

from . import DedupIndex, Params, fingerprint, gather_chunks, scan_sizes

PLACEMENTS = ("gpu_both", "gpu_dedup_cpu_compress", "cpu_dedup_gpu_compress", "cpu_both",
              "gpu_dedup_split")


@dataclass
class CpuArm:
    """The CPU side of the integration options (supplied by the caller).

    compress(x_u8, p) -> (out_u8, sizes_u32, offsets_u64, total): the method's
        result on the CPU (thread per chunk, §3.2(1));
    dedup(x_u8, chunk_size) -> (index_i64, unique_i32): first-occurrence
        indexing of the chunks' SHA-1 fingerprints (R17, R18);
    cores: host threads it uses (reported).
    """
    compress: Callable
    dedup: Callable
    cores: int


def _result(out, sizes, offsets, total, index, unique):
    return {"out": np.asarray(out)[: int(total)], "sizes": np.asarray(sizes, np.uint32),
            "offsets": np.asarray(offsets, np.uint64), "total": int(total),
            "index": np.asarray(index, np.int64), "unique": np.asarray(unique, np.int32)}


def _unique_host(x, C, unique):
    """Gather the unique chunks of a host stream in stream order."""
    n = x.size
    N = unique.size
    idx = np.flatnonzero(unique)
    if idx.size == 0:
        return np.zeros(0, np.uint8)
    parts = [x[i * C: min(n, (i + 1) * C)] for i in idx]
    return np.concatenate(parts) if len(parts) > 1 else parts[0].copy()


class Integrated:
    """Dedup-then-compress of host-resident streams under one placement.

    Device buffers (input, fingerprints, index, unique buffer, compression
    workspace) and pinned host staging are kept across calls and regrown when
    a longer stream arrives, so a placement's time is its data movement and
    kernels, not allocation."""

    def __init__(self, p: Params, cpu: CpuArm, device="cuda", split_fraction: float | None = None):
        import torch

        self.p = p
        self.cpu = cpu
        self.dev = torch.device(device)
        self.split_fraction = split_fraction
        self.rates = {}
        self._cap = 0

    def _ensure(self, n):
        import torch

        from . import Workspace

        if n <= self._cap:
            return
        C = self.p.chunk_size
        N = max(1, -(-n // C))
        with torch.cuda.device(self.dev):
            self.xd = torch.empty(n, dtype=torch.uint8, device=self.dev)
            self.ubuf = torch.empty(n, dtype=torch.uint8, device=self.dev)
            self.fp = torch.empty((N, 20), dtype=torch.uint8, device=self.dev)
            self.idx = torch.empty(N, dtype=torch.int64, device=self.dev)
            self.uniq = torch.empty(N, dtype=torch.int32, device=self.dev)
            self.rank = torch.empty(N, dtype=torch.int64, device=self.dev)
            self.index = DedupIndex.for_chunks(N, self.dev)
            self.ws = Workspace(n, self.p, self.dev)
        self.h_out = torch.empty(n, dtype=torch.uint8, pin_memory=True)
        self.h_in = torch.empty(n, dtype=torch.uint8, pin_memory=True)
        self._cap = n

    def _pinned(self, x):
        """The stream as a pinned host tensor (I/O buffers are pinned: a caller
        that passes one avoids the staging copy)."""
        import torch

        if isinstance(x, torch.Tensor) and x.is_pinned():
            return x
        t = self.h_in[: x.size]
        t.numpy()[:] = x
        return t

    # ---- the GPU pieces (this package's kernels) ---------------------------
    def _h2d(self, x):
        n = int(x.size if isinstance(x, np.ndarray) else x.numel())
        self._ensure(n)
        xd = self.xd[:n]
        xd.copy_(self._pinned(x), non_blocking=True)
        return xd

    def _gpu_dedup(self, xd):
        """-> (index, unique, gathered unique bytes), all on the device."""
        C = self.p.chunk_size
        n = xd.numel()
        N = -(-n // C)
        self.index.reset()
        fingerprint(xd, C, out=self.fp)
        self.index.index(self.fp[:N], 0, index=self.idx, unique=self.uniq)
        _, nu_t = scan_sizes(self.uniq[:N], 0, offsets=self.rank)
        nu = int(nu_t.item())
        ub = nu * C
        if N and bool(self.uniq[N - 1].item()) and n % C:
            ub -= C - n % C
        gather_chunks(xd, C, self.uniq[:N], self.rank[:N], self.ubuf)
        return self.idx[:N], self.uniq[:N], self.ubuf[:ub]

    def _gpu_compress(self, ud):
        from . import compress_compact, compress_encode

        n = ud.numel()
        N = -(-n // self.p.chunk_size)
        if n == 0:
            return np.zeros(0, np.uint8), np.zeros(0, np.uint32), np.zeros(0, np.uint64), 0
        compress_encode(ud, self.p, self.ws)
        compress_compact(ud, self.p, self.ws)
        sizes = self.ws.sizes[:N].cpu().numpy().view(np.uint32)
        offs = self.ws.offsets[:N].cpu().numpy().view(np.uint64)
        t = int(self.ws.total.item())
        ho = self.h_out[:t]
        ho.copy_(self.ws.out[:t])
        # a view of the pinned destage buffer: valid until the next run
        return ho.numpy(), sizes, offs, t

    # ---- placements ----------------------------------------------------------
    @staticmethod
    def _np(x):
        return x if isinstance(x, np.ndarray) else x.numpy()

    def run(self, x, placement: str) -> dict:
        """x: host uint8 stream (numpy array or CPU tensor, ideally pinned).
        Returns the placement-independent result; a GPU placement's "out" is a
        view of the pinned destage buffer, valid until the next run."""
        C = self.p.chunk_size
        if placement == "gpu_both":
            idx, uniq, ud = self._gpu_dedup(self._h2d(x))
            out, sizes, offs, tot = self._gpu_compress(ud)
            return _result(out, sizes, offs, tot, idx.cpu().numpy(), uniq.cpu().numpy())
        if placement == "gpu_dedup_cpu_compress":
            idx, uniq, ud = self._gpu_dedup(self._h2d(x))
            out, sizes, offs, tot = self.cpu.compress(ud.cpu().numpy(), self.p)
            return _result(out, sizes, offs, tot, idx.cpu().numpy(), uniq.cpu().numpy())
        if placement == "cpu_dedup_gpu_compress":
            idx, uniq = self.cpu.dedup(self._np(x), C)
            ub = _unique_host(self._np(x), C, uniq)
            if ub.size == 0:
                return _result(np.zeros(0, np.uint8), [], [], 0, idx, uniq)
            out, sizes, offs, tot = self._gpu_compress(self._h2d(ub))
            return _result(out, sizes, offs, tot, idx, uniq)
        if placement == "cpu_both":
            idx, uniq = self.cpu.dedup(self._np(x), C)
            out, sizes, offs, tot = self.cpu.compress(_unique_host(self._np(x), C, uniq), self.p)
            return _result(out, sizes, offs, tot, idx, uniq)
        if placement == "gpu_dedup_split":
            return self._run_split(x)
        raise ValueError(f"unknown placement {placement!r}")

    def _run_split(self, x):
        """GPU dedup; the unique chunks [0, k) compressed on the GPU while the
        CPU compresses [k, nu) concurrently; results concatenated in stream
        order (the CPU part's offsets shifted by the GPU part's total)."""
        C = self.p.chunk_size
        f = self.split_fraction if self.split_fraction is not None else 0.0
        idx, uniq, ud = self._gpu_dedup(self._h2d(x))
        nu = -(-ud.numel() // C)
        k = min(nu, max(0, int(round((1.0 - f) * nu))))
        cpu_part = ud[k * C:].cpu().numpy() if k < nu else np.zeros(0, np.uint8)
        res = {}

        def cpu_side():
            res["cpu"] = self.cpu.compress(cpu_part, self.p) if cpu_part.size else \
                (np.zeros(0, np.uint8), np.zeros(0, np.uint32), np.zeros(0, np.uint64), 0)

        th = threading.Thread(target=cpu_side)
        th.start()
        g = self._gpu_compress(ud[: k * C]) if k else \
            (np.zeros(0, np.uint8), np.zeros(0, np.uint32), np.zeros(0, np.uint64), 0)
        th.join()
        c = res["cpu"]
        out = np.concatenate([g[0], np.asarray(c[0])[: int(c[3])]])
        sizes = np.concatenate([g[1], c[1]]).astype(np.uint32)
        offs = np.concatenate([g[2], np.asarray(c[2], np.uint64) + np.uint64(g[3])]).astype(np.uint64)
        return _result(out, sizes, offs, g[3] + int(c[3]), idx.cpu().numpy(), uniq.cpu().numpy())

    # ---- the paper's selection by dummy I/O ------------------------------------
    def calibrate(self, dummy: np.ndarray, repeats: int = 2) -> dict:
        """Time every placement on a dummy stream (host in, host out) and pick
        the fastest.  The split fraction is set from the measured compression
        rates of the two processors (f = cpu / (cpu + gpu)) before the split
        placement is timed.  Returns {"gbs": {placement: GB/s}, "pick": name,
        "split_fraction": f}."""
        import torch

        n = int(dummy.size if isinstance(dummy, np.ndarray) else dummy.numel())
        if not (isinstance(dummy, torch.Tensor) and dummy.is_pinned()):  # I/O buffers are pinned
            pd = torch.empty(n, dtype=torch.uint8, pin_memory=True)
            pd.numpy()[:] = self._np(dummy)
            dummy = pd
        gbs = {}
        for pl in PLACEMENTS:
            if pl == "gpu_dedup_split":
                cpu_c = self.rates.get("cpu_compress")
                gpu_c = self.rates.get("gpu_compress")
                self.split_fraction = cpu_c / (cpu_c + gpu_c) if cpu_c and gpu_c else 0.0
            self.run(dummy, pl)  # warm-up (allocations, library loads)
            best = None
            for _ in range(repeats):
                torch.cuda.synchronize(self.dev)
                t0 = time.perf_counter()
                r = self.run(dummy, pl)
                torch.cuda.synchronize(self.dev)
                dt = time.perf_counter() - t0
                best = dt if best is None else min(best, dt)
            gbs[pl] = n / best / 1e9
            if pl == "gpu_dedup_cpu_compress":  # compression rates for the split
                ub = _unique_host(self._np(dummy), self.p.chunk_size, r["unique"])
                t0 = time.perf_counter()
                self.cpu.compress(ub, self.p)
                self.rates["cpu_compress"] = ub.size / (time.perf_counter() - t0)
                ud = self._h2d(ub)
                torch.cuda.synchronize(self.dev)
                t0 = time.perf_counter()
                self._gpu_compress(ud)
                torch.cuda.synchronize(self.dev)
                self.rates["gpu_compress"] = ub.size / (time.perf_counter() - t0)
        pick = max(gbs, key=gbs.get)
        return {"gbs": gbs, "pick": pick, "split_fraction": self.split_fraction}
