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
