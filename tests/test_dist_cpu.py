"""Multi-process (gloo, CPU) tests of the sharding / global-offset logic of
paper_conf_pact_map17_b200.dist.  The per-rank compression and
the scan are substituted by CPU stand-ins (the oracle and numpy) so the
host-side plumbing -- contiguous shards with the remainder on the first ranks,
zero-padded all-gather of per-chunk sizes, global offsets from one exclusive
scan -- is checked end to end without a GPU.  The CUDA path itself is covered
by the gpu tests; the product path never uses these stand-ins."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_pact_map17_b200.dist import ShardedCompressor, max_shard, shard_range


def test_shard_range_partition():
    for N in [0, 1, 7, 8, 9, 100, 4_194_304]:
        for R in [1, 2, 3, 4, 8]:
            rs = [shard_range(N, R, r) for r in range(R)]
            assert rs[0][0] == 0 and rs[-1][1] == N
            for (a, b), (c, d) in zip(rs, rs[1:]):
                assert b == c
            sizes = [b - a for a, b in rs]
            assert max(sizes) - min(sizes) <= 1 and max(sizes) <= max_shard(N, R)
            assert sizes == sorted(sizes, reverse=True)


class OracleOps:
    """CPU stand-in for CudaOps (test only)."""

    def __init__(self, p):
        import oracle

        self.ref = oracle
        self.rp = oracle.Params(chunk_size=p.chunk_size, parse=p.parse)

    def compress(self, x):
        out, sizes, offs, total = self.ref.compress(x.numpy(), self.rp, n_threads=1)
        return (torch.from_numpy(out.copy()), torch.from_numpy(sizes.view(np.int32).copy()),
                torch.tensor([total], dtype=torch.int64))

    def scan(self, sizes_all, offsets, total):
        s = sizes_all.numpy().view(np.uint32).astype(np.uint64)
        ex = np.concatenate([[0], np.cumsum(s[:-1])]).astype(np.uint64)
        offsets.copy_(torch.from_numpy(ex.view(np.int64)))
        total.fill_(int(s.sum()))

    def all_gather(self, out, inp, group):
        try:
            dist.all_gather_into_tensor(out, inp, group=group)
        except (RuntimeError, NotImplementedError):
            parts = list(out.chunk(dist.get_world_size(group)))
            dist.all_gather(parts, inp, group=group)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, n_global, C, q, parse=0):
    import synth
    import paper_conf_pact_map17_b200 as lzr

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        p = lzr.Params(chunk_size=C, parse=parse)
        sc = ShardedCompressor(n_global, p, None, "cpu", ops=OracleOps(p))
        x_local = synth.fill_host(sc.n_local, C, "mix", seed=77, first_chunk=sc.lo) if sc.n_local else np.zeros(0, np.uint8)
        res = sc(torch.from_numpy(np.ascontiguousarray(x_local)))
        nl = sc.hi - sc.lo
        q.put((rank, sc.lo, sc.hi, res.global_offsets().numpy().copy(),
               int(res.global_total.item()), res.out[: int(res.local_total.item())].numpy().copy() if nl else np.zeros(0, np.uint8),
               res.sizes_all.numpy().copy()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,nchunks,tail,parse", [(2, 37, 100, 0), (3, 10, 0, 0), (4, 3, 17, 0), (2, 1, 5, 0),
                                                     (2, 37, 100, 1)])
def test_sharded_offsets_match_single_process(ref, world, nchunks, tail, parse):
    import synth

    C = 512
    n_global = nchunks * C + tail if tail else nchunks * C
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, n_global, C, q, parse)) for r in range(world)]
    for pr in procs:
        pr.start()
    results = [q.get(timeout=120) for _ in range(world)]
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    x = synth.fill_host(n_global, C, "mix", seed=77)
    r_out, r_sizes, r_offs, r_tot = ref.compress(x, ref.Params(chunk_size=C, parse=parse))
    N = ref.num_chunks(n_global, ref.Params(chunk_size=C))
    for rank, lo, hi, goffs, gtot, out_local, sizes_all in sorted(results, key=lambda t: t[0]):
        assert gtot == r_tot
        assert np.array_equal(goffs.view(np.uint64), r_offs[lo:hi])
        if hi > lo:
            a = int(r_offs[lo])
            assert out_local.tobytes() == r_out[a: a + out_local.size].tobytes()
        # gathered sizes, de-padded, are the global sizes in chunk order
        mx = max_shard(N, world)
        got = np.concatenate([sizes_all.view(np.uint32)[r * mx: r * mx + (shard_range(N, world, r)[1] - shard_range(N, world, r)[0])]
                              for r in range(world)])
        assert np.array_equal(got, r_sizes)


# ---- multi-rank dedup (ShardedDedup): host-side routing over gloo -----------------
class OracleDedupOps:
    """CPU stand-in for CudaDedupOps (test only): oracle fingerprints, a numpy
    owner partition and router, and a dict index with insert-or-min semantics."""

    def __init__(self):
        import oracle

        self.ref = oracle
        self.table = {}

    def fingerprint(self, x, C):
        return torch.from_numpy(self.ref.fingerprints(x.numpy(), C, n_threads=1).copy())

    @staticmethod
    def _owner(fp, R):
        w2 = (fp[:, 8].astype(np.uint64) << 24) | (fp[:, 9].astype(np.uint64) << 16) | \
             (fp[:, 10].astype(np.uint64) << 8) | fp[:, 11].astype(np.uint64)
        return ((w2 * np.uint64(R)) >> np.uint64(32)).astype(np.int64)

    def owner_counts(self, fp, R):
        return torch.from_numpy(np.bincount(self._owner(fp.numpy(), R), minlength=R).astype(np.int32))

    def route(self, fp, first, R, base):
        f = fp.numpy()
        own = self._owner(f, R)
        order = np.argsort(own, kind="stable")
        slot = np.empty(len(f), np.int32)
        slot[order] = np.arange(len(f), dtype=np.int32)
        gidx = first + np.arange(len(f), dtype=np.int64)
        return torch.from_numpy(f[order].copy()), torch.from_numpy(gidx[order].copy()), torch.from_numpy(slot)

    def index_gidx(self, fp, gidx):
        f, g = fp.numpy(), gidx.numpy()
        for k in range(len(f)):  # insert-or-min over the whole batch first
            key = f[k].tobytes()
            self.table[key] = min(self.table.get(key, int(g[k])), int(g[k]))
        return torch.tensor([self.table[f[k].tobytes()] for k in range(len(f))], dtype=torch.int64)

    def unroute(self, back, slot, first):
        idx = back.numpy()[slot.numpy()]
        uniq = (idx == first + np.arange(len(idx))).astype(np.int32)
        return torch.from_numpy(idx.copy()), torch.from_numpy(uniq)

    def all_to_all(self, out, inp, out_splits, in_splits, group):
        dist.all_to_all_single(out, inp, output_split_sizes=out_splits, input_split_sizes=in_splits,
                               group=group)


def _dedup_worker(rank, world, port, n_chunks, C, rounds, q):
    """The stream is indexed in `rounds` global batches (stream order); each
    batch is sharded over the ranks by contiguous chunk ranges."""
    import synth
    from paper_conf_pact_map17_b200.dist import ShardedDedup

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        x = synth.fill_host(n_chunks * C, C, "mix_dedup")
        per = -(-n_chunks // rounds)
        sd = ShardedDedup(per, ops=OracleDedupOps())
        outs = []
        for b in range(rounds):
            g0, g1 = b * per, min(n_chunks, (b + 1) * per)
            lo, hi = shard_range(g1 - g0, world, rank)
            lo, hi = g0 + lo, g0 + hi
            _, idx, un = sd(torch.from_numpy(np.ascontiguousarray(x[lo * C:hi * C])), C, lo)
            outs.append((lo, idx.numpy().copy(), un.numpy().copy()))
        q.put((rank, outs))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,rounds", [(2, 1), (3, 1), (2, 3), (4, 2)])
def test_sharded_dedup_matches_single_process(ref, world, rounds):
    import synth

    C, n_chunks = 256, 300
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_dedup_worker, args=(r, world, port, n_chunks, C, rounds, q))
             for r in range(world)]
    for pr in procs:
        pr.start()
    results = [q.get(timeout=180) for _ in range(world)]
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    x = synth.fill_host(n_chunks * C, C, "mix_dedup")
    r_idx, r_hit, _ = ref.dedup_index(ref.fingerprints(x, C), 0)
    assert r_hit.sum() > 0.3 * n_chunks  # the stream does carry cross-shard duplicates
    got_idx = np.zeros(n_chunks, np.int64) - 1
    got_un = np.zeros(n_chunks, np.int32) - 1
    for rank, outs in results:
        for b0, idx, un in outs:
            got_idx[b0:b0 + len(idx)] = idx
            got_un[b0:b0 + len(un)] = un
    assert np.array_equal(got_idx.astype(np.uint64), r_idx)
    assert np.array_equal(got_un.astype(bool), ~r_hit.astype(bool))
