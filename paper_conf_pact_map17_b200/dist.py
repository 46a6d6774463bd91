"""Multi-GPU sharding of chunk batches.

Chunks are independent (§3.2(1) "there is no data dependency between
chunks"), so rank r of R compresses a contiguous chunk range on its own GPU.
The only exchange step is the one the global layout needs: every rank
all-gathers the per-chunk uint32 compressed sizes (NCCL over NVLink /
NVSwitch) and derives the global offsets with the device scan of liblzr
(``lzr_scan_sizes``).  Compressed bytes never leave their rank.

Shards are padded to ceil(N/R) chunks with zero sizes, so the gathered array
is [R, ceil(N/R)] and its exclusive scan directly gives every real chunk's
global offset (padding contributes 0) -- no reshuffle on the data path.

The compress / scan / collective steps are taken from an ``ops`` object; the
default is the CUDA path (liblzr) with ``torch.distributed`` collectives.
Tests substitute a CPU implementation to exercise the host-side shard and
offset logic over a gloo group; there is no CPU fallback in the product path.
"""
from __future__ import annotations

from contextlib import nullcontext
from dataclasses import dataclass

import torch
import torch.distributed as dist

from . import (DedupIndex, Params, Workspace, compress, fingerprint, num_chunks, owner_counts, route,
               scan_sizes, unroute)


def shard_range(n_chunks: int, world: int, rank: int) -> tuple[int, int]:
    """Contiguous chunk range [lo, hi) of `rank`; the remainder goes to the first ranks."""
    base, rem = divmod(n_chunks, world)
    lo = rank * base + min(rank, rem)
    return lo, lo + base + (1 if rank < rem else 0)


def max_shard(n_chunks: int, world: int) -> int:
    return -(-n_chunks // world)


def _staged(group) -> bool:
    """True when the group's backend cannot take CUDA tensors in the exchange
    collectives (gloo): the tensors are then staged through host memory.  The
    data-path backend of the product is NCCL; gloo serves several ranks that
    share one GPU (tests, bench --backend gloo)."""
    return dist.get_backend(group) != "nccl"


def all_gather_into(out: torch.Tensor, inp: torch.Tensor, group=None) -> None:
    """all_gather_into_tensor on NCCL; host-staged all_gather on gloo."""
    if not _staged(group) or not out.is_cuda:
        try:
            dist.all_gather_into_tensor(out, inp, group=group)
            return
        except (RuntimeError, NotImplementedError):
            if out.is_cuda:
                raise
    o = torch.empty(out.shape, dtype=out.dtype)
    dist.all_gather(list(o.chunk(dist.get_world_size(group))), inp.cpu(), group=group)
    out.copy_(o)


def all_to_all_into(out: torch.Tensor, inp: torch.Tensor, out_splits, in_splits, group=None) -> None:
    """all_to_all_single on NCCL; host-staged on gloo."""
    if not _staged(group) or not out.is_cuda:
        dist.all_to_all_single(out, inp, output_split_sizes=out_splits,
                               input_split_sizes=in_splits, group=group)
        return
    o = torch.empty(out.shape, dtype=out.dtype)
    dist.all_to_all_single(o, inp.cpu(), output_split_sizes=out_splits,
                           input_split_sizes=in_splits, group=group)
    out.copy_(o)


def _on(device):
    """Make `device` current around liblzr calls (the C ABI works on the
    current device, include/lzr.h)."""
    dev = torch.device(device) if device is not None else None
    return torch.cuda.device(dev) if dev is not None and dev.type == "cuda" else nullcontext()


class CudaOps:
    """The product path: liblzr kernels + torch.distributed collectives."""

    def __init__(self, p: Params, n_local: int, device):
        self.p = p
        self.device = device
        with _on(device):
            self.ws = Workspace(n_local, p, device)

    def bind_sizes(self, sizes_pad):
        # the encoder writes the per-chunk sizes straight into the padded
        # all-gather input (no copy on the data path)
        assert sizes_pad.numel() >= self.ws.N
        self.ws.sizes = sizes_pad

    def compress(self, x):
        with _on(x.device):
            out, sizes, offsets, total = compress(x, self.p, ws=self.ws)
        return out, sizes, total

    def scan(self, sizes_all, offsets, total):
        with _on(sizes_all.device):
            scan_sizes(sizes_all, 0, offsets=offsets, total=total)

    def all_gather(self, out, inp, group):
        all_gather_into(out, inp, group)


@dataclass
class ShardResult:
    out: torch.Tensor            # local compacted streams (first local_total bytes valid)
    local_sizes: torch.Tensor    # [N_r] int32
    local_total: torch.Tensor    # [1] int64
    sizes_all: torch.Tensor      # [R * maxN] int32, zero-padded per rank
    offsets_all: torch.Tensor    # [R * maxN] int64 global exclusive offsets
    global_total: torch.Tensor   # [1] int64
    lo: int                      # this rank's chunk range [lo, hi) of the global stream
    hi: int
    max_n: int                   # padded shard length (ceil(N / R))
    rank: int                    # this rank in the group (row of sizes_all / offsets_all)

    def global_offsets(self) -> torch.Tensor:
        """Global offsets of this rank's chunks (view)."""
        r = self.rank
        return self.offsets_all[r * self.max_n: r * self.max_n + (self.hi - self.lo)]


class ShardedCompressor:
    """compress_sharded with persistent buffers (one instance per rank)."""

    def __init__(self, n_bytes_global: int, p: Params, group=None, device=None, ops=None):
        self.group = group
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        self.p = p
        self.N = num_chunks(n_bytes_global, p)
        self.n_global = n_bytes_global
        self.lo, self.hi = shard_range(self.N, self.world, self.rank)
        self.max_n = max(1, max_shard(self.N, self.world))
        self.byte_lo = self.lo * p.chunk_size
        self.byte_hi = min(n_bytes_global, self.hi * p.chunk_size)
        self.n_local = self.byte_hi - self.byte_lo
        dev = torch.device(device) if device is not None else None
        self.ops = ops if ops is not None else CudaOps(p, self.n_local, dev)
        kw = dict(device=dev) if dev is not None else {}
        self.sizes_pad = torch.zeros(self.max_n, dtype=torch.int32, **kw)
        self.sizes_all = torch.zeros(self.world * self.max_n, dtype=torch.int32, **kw)
        self.offsets_all = torch.zeros(self.world * self.max_n, dtype=torch.int64, **kw)
        self.global_total = torch.zeros(1, dtype=torch.int64, **kw)
        if hasattr(self.ops, "bind_sizes"):
            self.ops.bind_sizes(self.sizes_pad)

    def __call__(self, x_local) -> ShardResult:
        """x_local: this rank's bytes [byte_lo, byte_hi) of the global stream."""
        assert x_local.numel() == self.n_local
        nl = self.hi - self.lo
        if nl:
            out, sizes, total = self.ops.compress(x_local)
            if sizes.data_ptr() != self.sizes_pad.data_ptr():
                self.sizes_pad[:nl].copy_(sizes[:nl])
        else:
            out = x_local.new_empty(0)
            sizes = self.sizes_pad[:0]
            total = torch.zeros(1, dtype=torch.int64, device=self.sizes_pad.device)
        self.ops.all_gather(self.sizes_all, self.sizes_pad, self.group)
        self.ops.scan(self.sizes_all, self.offsets_all, self.global_total)
        return ShardResult(out, sizes[:nl], total, self.sizes_all, self.offsets_all,
                           self.global_total, self.lo, self.hi, self.max_n, self.rank)


def compress_sharded(x_local, p: Params, n_bytes_global: int, group=None):
    """One-shot convenience wrapper (allocates buffers every call)."""
    return ShardedCompressor(n_bytes_global, p, group, x_local.device)(x_local)


# ---- multi-GPU dedup (SURVEY.md §8(f) N2 across ranks) ------------
class CudaDedupOps:
    """The product path of ShardedDedup: liblzr kernels + torch.distributed."""

    def __init__(self, index: DedupIndex):
        self.index = index

    def fingerprint(self, x, C):
        with _on(x.device):
            return fingerprint(x, C)

    def owner_counts(self, fp, R):
        with _on(fp.device):
            return owner_counts(fp, R)

    def route(self, fp, first, R, base):
        with _on(fp.device):
            return route(fp, first, R, base)

    def index_gidx(self, fp, gidx):
        with _on(fp.device):
            return self.index.index_gidx(fp, gidx)[0]

    def unroute(self, back, slot, first):
        with _on(slot.device):
            return unroute(back, slot, first)

    def all_to_all(self, out, inp, out_splits, in_splits, group):
        all_to_all_into(out, inp, out_splits, in_splits, group)


class ShardedDedup:
    """Global dedup of a stream sharded over R ranks (contiguous chunk ranges).

    The index is partitioned over the ranks by fingerprint (owner = third
    fingerprint word scaled to R; §3.1(1) bins, spread over GPUs).  One
    call: fingerprint the local chunks; count and route (fingerprint, global
    chunk index) records to their owners (all-to-all of the counts, then of the
    records: the real exchange step of dedup); each owner inserts and looks up
    everything it received in its own DedupIndex (insert-or-min, so the index
    number = the first occurrence in the global stream, wherever it lives);
    the index numbers go back by the reverse all-to-all and are put back in
    chunk order.  Result per local chunk: (index number, unique flag) equal to
    single-process indexing of the whole stream (R18).
    """

    def __init__(self, n_local_max: int, group=None, device=None, ops=None, bin_slots: int = 64,
                 skew: float = 1.5):
        self.group = group
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        if ops is None:
            # an owner receives ~n_local chunks on average; skew covers imbalance
            cap = int(skew * max(1, n_local_max)) + 1024
            with _on(device):
                ops = CudaDedupOps(DedupIndex.for_chunks(cap, device, bin_slots))
        self.ops = ops

    def __call__(self, x_local, chunk_size: int, first_chunk: int):
        R = self.world
        fp = self.ops.fingerprint(x_local, chunk_size)
        N = fp.shape[0]
        dev = fp.device
        counts = self.ops.owner_counts(fp, R).to(torch.int64)
        recv_counts = torch.empty_like(counts)
        self.ops.all_to_all(recv_counts, counts, None, None, self.group)
        in_splits = counts.cpu().tolist()
        out_splits = recv_counts.cpu().tolist()
        base = torch.zeros(R, dtype=torch.int64, device=dev)
        if R > 1:
            base[1:] = torch.cumsum(counts, 0)[:-1]
        send_fp, send_gidx, slot = self.ops.route(fp, first_chunk, R, base)
        n_recv = int(sum(out_splits))
        recv_fp = torch.empty((n_recv, 20), dtype=torch.uint8, device=dev)
        recv_gidx = torch.empty(n_recv, dtype=torch.int64, device=dev)
        self.ops.all_to_all(recv_fp, send_fp, out_splits, in_splits, self.group)
        self.ops.all_to_all(recv_gidx, send_gidx, out_splits, in_splits, self.group)
        recv_index = self.ops.index_gidx(recv_fp, recv_gidx) if n_recv else recv_gidx
        back = torch.empty(N, dtype=torch.int64, device=dev)
        self.ops.all_to_all(back, recv_index, in_splits, out_splits, self.group)
        index, unique = self.ops.unroute(back, slot, first_chunk)
        return fp, index, unique
