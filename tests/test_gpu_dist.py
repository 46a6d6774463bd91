"""The sharded path on the GPU: ShardedCompressor with the CUDA ops over a real
NCCL process group (world size 1 -- the pool gives one GPU per call), checked
against the single-call path and the oracle's global offsets.  The multi-rank
host logic is covered with gloo in tests/test_dist_cpu.py."""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_sharded_nccl_world1(ref):
    import torch.distributed as dist

    import __graft_entry__
    __graft_entry__.build()
    import synth
    import paper_conf_pact_map17_b200 as lzr
    from paper_conf_pact_map17_b200.dist import ShardedCompressor

    assert torch.cuda.is_available()
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(_port())
    dev = torch.device("cuda", 0)
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=dev)
    try:
        n = 4096 * 300 + 123
        p = lzr.Params()
        sc = ShardedCompressor(n, p, None, dev)
        x = torch.empty(n, dtype=torch.uint8, device=dev)
        synth.fill_device(x, 4096, "mix", first_chunk=sc.lo)
        res = sc(x)
        torch.cuda.synchronize()
        r_out, r_sizes, r_offs, r_tot = ref.compress(x.cpu().numpy(), ref.Params())
        assert int(res.global_total.item()) == r_tot
        assert np.array_equal(res.global_offsets().cpu().numpy().view(np.uint64), r_offs)
        assert np.array_equal(res.local_sizes.cpu().numpy().view(np.uint32), r_sizes)
        assert np.array_equal(res.out[:r_tot].cpu().numpy(), r_out)
    finally:
        dist.destroy_process_group()


def test_sharded_dedup_nccl_world1(ref):
    """ShardedDedup with the CUDA ops over NCCL (world 1): all-to-all of counts,
    records and index numbers, owner-side insert/lookup, unroute."""
    import torch.distributed as dist

    import __graft_entry__
    __graft_entry__.build()
    import synth
    from paper_conf_pact_map17_b200.dist import ShardedDedup

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(_port())
    dev = torch.device("cuda", 0)
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=dev)
    try:
        C, N = 4096, 3000
        x = torch.empty(N * C, dtype=torch.uint8, device=dev)
        synth.fill_device(x, C, "mix_dedup")
        sd = ShardedDedup(N, device=dev)
        h = N // 2  # two batches in stream order
        _, i0, u0 = sd(x[: h * C], C, 0)
        _, i1, u1 = sd(x[h * C:], C, h)
        torch.cuda.synchronize()
        r_idx, r_hit, _ = ref.dedup_index(ref.fingerprints(x.cpu().numpy(), C), 0)
        got = np.concatenate([i0.cpu().numpy(), i1.cpu().numpy()]).view(np.uint64)
        un = np.concatenate([u0.cpu().numpy(), u1.cpu().numpy()])
        assert np.array_equal(got, r_idx)
        assert np.array_equal(un.astype(bool), ~r_hit.astype(bool))
    finally:
        dist.destroy_process_group()


def test_dedup_routing_kernels_emulated_ranks(ref):
    """The routing kernels with R = 3 owners, the exchange emulated in one
    process: every simulated rank routes its shard, each owner indexes what it
    receives from all ranks (its own table), results are sent back and
    unrouted; must equal single-process first-occurrence indexing."""
    import __graft_entry__
    __graft_entry__.build()
    import synth
    import paper_conf_pact_map17_b200 as lzr
    from paper_conf_pact_map17_b200.dist import shard_range

    dev = torch.device("cuda", 0)
    C, N, R = 4096, 2500, 3
    x = torch.empty(N * C, dtype=torch.uint8, device=dev)
    synth.fill_device(x, C, "mix_dedup")
    owners = [lzr.DedupIndex.for_chunks(N, dev) for _ in range(R)]
    sent = []
    for r in range(R):
        lo, hi = shard_range(N, R, r)
        fp = lzr.fingerprint(x[lo * C: hi * C], C)
        cnt = lzr.owner_counts(fp, R).to(torch.int64)
        base = torch.zeros(R, dtype=torch.int64, device=dev)
        base[1:] = torch.cumsum(cnt, 0)[:-1]
        sfp, sg, slot = lzr.route(fp, lo, R, base)
        sent.append((lo, hi, cnt.cpu().tolist(), base.cpu().tolist(), sfp, sg, slot))
    # owner o receives, from every rank r, that rank's block for o
    back = [torch.empty(hi - lo, dtype=torch.int64, device=dev) for lo, hi, *_ in sent]
    for o in range(R):
        blocks = [(r, s[3][o], s[2][o]) for r, s in enumerate(sent)]
        rfp = torch.cat([sent[r][4][b:b + c] for r, b, c in blocks])
        rg = torch.cat([sent[r][5][b:b + c] for r, b, c in blocks])
        ri = owners[o].index_gidx(rfp, rg)[0] if rfp.shape[0] else rg
        k = 0
        for r, b, c in blocks:
            back[r][b:b + c] = ri[k:k + c]
            k += c
    got_i, got_u = [], []
    for r, (lo, hi, *_rest) in enumerate(sent):
        idx, un = lzr.unroute(back[r], sent[r][6], lo)
        got_i.append(idx.cpu().numpy())
        got_u.append(un.cpu().numpy())
    for o in owners:
        assert int(o.overflow.item()) == 0
    r_idx, r_hit, _ = ref.dedup_index(ref.fingerprints(x.cpu().numpy(), C), 0)
    assert np.array_equal(np.concatenate(got_i).view(np.uint64), r_idx)
    assert np.array_equal(np.concatenate(got_u).astype(bool), ~r_hit.astype(bool))


# ---- several ranks on the real kernels ---------------------------------------
# The pool gives one GPU per call, and NCCL refuses two ranks on one device, so
# these run R processes on cuda:0 over a gloo group: the product ops (CudaOps /
# CudaDedupOps: liblzr kernels) with the exchange tensors staged through host
# memory (dist.all_gather_into / all_to_all_into).  Uneven shards exercise the
# zero padding of the size all-gather and the global scan over R * ceil(N/R).
def _mp_compress_worker(rank, world, port, n_global, C, parse, q):
    import torch.distributed as dist

    import synth
    import paper_conf_pact_map17_b200 as lzr
    from paper_conf_pact_map17_b200.dist import ShardedCompressor

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        p = lzr.Params(chunk_size=C, parse=parse)
        sc = ShardedCompressor(n_global, p, None, dev)
        x = torch.empty(sc.n_local, dtype=torch.uint8, device=dev)
        if sc.n_local:
            synth.fill_device(x, C, "mix", first_chunk=sc.lo)
        res = sc(x)
        torch.cuda.synchronize()
        lt = int(res.local_total.item())
        q.put((rank, sc.lo, sc.hi, sc.max_n, res.rank, res.global_offsets().cpu().numpy().copy(),
               int(res.global_total.item()), res.out[:lt].cpu().numpy().copy(),
               res.local_sizes.cpu().numpy().copy(), res.sizes_all.cpu().numpy().copy()))
    except Exception as e:  # surface the failure to the parent
        q.put((rank, repr(e)))
        raise
    finally:
        dist.destroy_process_group()


def _spawn(target, world, args, timeout=300):
    import torch.multiprocessing as mp

    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=target, args=(r, world, port, *args, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    res = [q.get(timeout=timeout) for _ in range(world)]
    for pr in procs:
        pr.join(timeout=60)
    for r in res:
        assert len(r) > 2, f"rank {r[0]} failed: {r[1]}"
    for pr in procs:
        assert pr.exitcode == 0
    return sorted(res, key=lambda t: t[0])


@pytest.mark.parametrize("world,nchunks,tail,C,parse", [(2, 301, 123, 4096, 0), (3, 100, 0, 4096, 0),
                                                       (3, 7, 5, 8192, 0), (2, 55, 77, 4096, 1),
                                                       (4, 3, 0, 4096, 0)])
def test_sharded_real_kernels_multirank(ref, world, nchunks, tail, C, parse):
    """ShardedCompressor with the CUDA ops at world 2-4 (uneven shards, a rank
    with no chunk at world 4 / 3 chunks) == the oracle over the whole stream:
    global offsets, total, gathered sizes and every rank's compacted bytes."""
    import __graft_entry__
    __graft_entry__.build()
    import synth
    from paper_conf_pact_map17_b200.dist import max_shard, shard_range

    n_global = nchunks * C + tail
    res = _spawn(_mp_compress_worker, world, (n_global, C, parse))
    x = synth.fill_host(n_global, C, "mix")
    r_out, r_sizes, r_offs, r_tot = ref.compress(x, ref.Params(chunk_size=C, parse=parse))
    N = r_sizes.size
    mx = max_shard(N, world)
    for rank, lo, hi, max_n, rrank, goffs, gtot, out_local, lsizes, sizes_all in res:
        assert (lo, hi) == shard_range(N, world, rank) and rrank == rank and max_n == mx
        assert gtot == r_tot
        assert np.array_equal(goffs.view(np.uint64), r_offs[lo:hi])
        assert np.array_equal(lsizes.view(np.uint32), r_sizes[lo:hi])
        if hi > lo:
            a = int(r_offs[lo])
            assert out_local.tobytes() == r_out[a: a + out_local.size].tobytes()
        sa = sizes_all.view(np.uint32)
        got = np.concatenate([sa[r * mx: r * mx + (shard_range(N, world, r)[1] - shard_range(N, world, r)[0])]
                              for r in range(world)])
        assert np.array_equal(got, r_sizes)
        pads = np.concatenate([sa[r * mx + (shard_range(N, world, r)[1] - shard_range(N, world, r)[0]):(r + 1) * mx]
                               for r in range(world)])
        assert not pads.any()


def _mp_dedup_worker(rank, world, port, n_chunks, C, rounds, q):
    import torch.distributed as dist

    import synth
    from paper_conf_pact_map17_b200.dist import ShardedDedup, shard_range

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        xh = synth.fill_host(n_chunks * C, C, "mix_dedup")
        per = -(-n_chunks // rounds)
        sd = ShardedDedup(per, device=dev)
        outs = []
        for b in range(rounds):
            g0, g1 = b * per, min(n_chunks, (b + 1) * per)
            lo, hi = shard_range(g1 - g0, world, rank)
            lo, hi = g0 + lo, g0 + hi
            x = torch.from_numpy(np.ascontiguousarray(xh[lo * C:hi * C])).to(dev)
            _, idx, un = sd(x, C, lo)
            torch.cuda.synchronize()
            outs.append((lo, idx.cpu().numpy().copy(), un.cpu().numpy().copy()))
        assert int(sd.ops.index.overflow.item()) == 0
        q.put((rank, outs, None))
    except Exception as e:
        q.put((rank, repr(e)))
        raise
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,rounds", [(2, 1), (3, 2)])
def test_sharded_dedup_real_kernels_multirank(ref, world, rounds):
    """ShardedDedup with the CUDA ops at world 2-3: fingerprints routed to their
    owner rank, owner-side insert-or-min, index numbers back; == single-process
    first-occurrence indexing of the whole stream (R18)."""
    import __graft_entry__
    __graft_entry__.build()
    import synth

    C, n_chunks = 4096, 1500
    res = _spawn(_mp_dedup_worker, world, (n_chunks, C, rounds))
    x = synth.fill_host(n_chunks * C, C, "mix_dedup")
    r_idx, r_hit, _ = ref.dedup_index(ref.fingerprints(x, C), 0)
    got_idx = np.zeros(n_chunks, np.int64) - 1
    got_un = np.zeros(n_chunks, np.int32) - 1
    for rank, outs, _ in res:
        for b0, idx, un in outs:
            got_idx[b0:b0 + len(idx)] = idx
            got_un[b0:b0 + len(un)] = un
    assert np.array_equal(got_idx.astype(np.uint64), r_idx)
    assert np.array_equal(got_un.astype(bool), ~r_hit.astype(bool))


def _bench_line(args, timeout=900):
    import json
    import subprocess
    import sys

    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, os.path.join(root, "bench.py"), *args], capture_output=True,
                       text=True, timeout=timeout, cwd=root)
    assert r.returncode == 0, r.stderr[-3000:]
    return json.loads(r.stdout.strip().splitlines()[-1])


def test_bench_gpus2_self_launch_gloo():
    """`bench.py --gpus 2` without torchrun starts 2 ranks itself (gloo, both on
    the one GPU): the line says n_gpus 2, covers both shards, round trip ok."""
    d = _bench_line(["--gpus", "2", "--backend", "gloo", "--bytes-per-rank", str(16 << 20),
                     "--steps", "3", "--warmup", "3", "--no-cpu", "--no-e2e", "--no-per-class"])
    assert d["n_gpus"] == 2 and len(d["per_rank_ms"]) == 2
    assert d["config"]["global_bytes"] == 2 * (16 << 20)
    assert d["decode"]["round_trip"] == "ok"
    assert "dp2" in d["config"]["parallelism"]


def test_bench_config5_gpus2_gloo():
    d = _bench_line(["--config", "5", "--gpus", "2", "--backend", "gloo", "--bytes-per-rank",
                     str(32 << 20), "--steps", "3", "--warmup", "3", "--no-cpu"])
    assert d["n_gpus"] == 2 and len(d["per_rank_ms"]) == 2
    assert 1.8 < d["config"]["dedup_ratio"] < 2.2
