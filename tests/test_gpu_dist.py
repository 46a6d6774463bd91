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
