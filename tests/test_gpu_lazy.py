"""GPU parity of the one-step lazy parse (R21)
against the oracle's lazy parse, byte for byte through the C ABI, on the same
inputs as the greedy parity tests: every stream class, the adversarial set
(runs, periods, small alphabets, ragged tails), a (C, W, m, M) grid incl.
W < C and C up to 32 KiB, and the full 256 MiB config-2 stream (sampled)."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

pytestmark = pytest.mark.gpu

import synth  # noqa: E402
from tests.test_gpu_parity import _adversarial, _check_full, lzr  # noqa: E402,F401


def _lazy(lzr, **kw):
    return lzr.Params(parse=lzr.PARSE_LAZY, **kw)


@pytest.mark.parametrize("cls", ["mix", "text", "random", "zeroruns", "cr2"])
def test_lazy_classes_bitexact(lzr, ref, cls):
    x = synth.fill_host(1 << 20, 4096, cls, seed=23)
    g_out, g_sizes, _ = _check_full(lzr, ref, x, _lazy(lzr))
    if cls in ("mix", "text"):
        # the lazy parse really differs from the greedy one on these streams
        _, greedy_sizes, _ = _check_full(lzr, ref, x, lzr.Params(), roundtrip=False)
        assert not np.array_equal(g_sizes, greedy_sizes)


@pytest.mark.parametrize("name,x", list(_adversarial()), ids=lambda v: v if isinstance(v, str) else "")
def test_lazy_adversarial_bitexact(lzr, ref, name, x):
    _check_full(lzr, ref, x, _lazy(lzr))


@pytest.mark.parametrize("C,W,m,M", [
    (4096, 4096, 3, 258), (4096, 4096, 5, 40), (4096, 4096, 3, 3), (4096, 4096, 4, 5),
    (4096, 1000, 4, 259), (4096, 1, 4, 259), (4096, 33, 6, 261), (16, 16, 3, 258), (528, 300, 4, 20),
    (8192, 8192, 4, 259), (8192, 2048, 4, 259), (16384, 16384, 4, 259), (32768, 32768, 4, 259),
    (65536, 65536, 4, 259), (65536, 30000, 3, 200),
])
def test_lazy_param_grid_bitexact(lzr, ref, C, W, m, M):
    n = max(C * 3 + C // 3 + 1, 3000)
    x = synth.fill_host(n, C, "mix", seed=C + W + m + M + 1)
    _check_full(lzr, ref, x, _lazy(lzr, chunk_size=C, window=W, min_match=m, max_match=M))


def test_lazy_config2_full_size_sampled(lzr, ref):
    """256 MiB mix, lazy, the launch configuration bench.py --parse lazy
    times: every 256th chunk + first/last 64 vs the oracle; full round trip."""
    n = 256 << 20
    p = _lazy(lzr)
    xd = torch.empty(n, dtype=torch.uint8, device="cuda")
    synth.fill_device(xd, 4096, "mix")
    out, sizes, offs, total = lzr.compress(xd, p)
    torch.cuda.synchronize()
    N = n // 4096
    idx = sorted(set(range(0, N, 256)) | set(range(64)) | set(range(N - 64, N)))
    g_sizes = sizes.cpu().numpy().view(np.uint32)
    g_offs = offs.cpu().numpy().view(np.uint64)
    g_out = out.cpu().numpy()
    r_streams, r_sizes = ref.compress_sampled(xd.cpu().numpy(), ref.Params(parse=1), idx)
    for k, i in enumerate(idx):
        assert g_sizes[i] == r_sizes[k], i
        assert g_out[g_offs[i]: g_offs[i] + g_sizes[i]].tobytes() == r_streams[k], i
    y, err = lzr.decompress(out, sizes, offs, n, p)
    torch.cuda.synchronize()
    assert int(err.item()) == 0 and torch.equal(y, xd)


def test_lazy_config2_every_chunk_vs_oracle(lzr, ref):
    """The lazy parse over all 65,536 chunks of the 256 MiB mix stream vs the
    oracle itself (thread per chunk on the host cores), every byte."""
    import os

    n = 256 << 20
    p = _lazy(lzr)
    xd = torch.empty(n, dtype=torch.uint8, device="cuda")
    synth.fill_device(xd, 4096, "mix")
    out, sizes, offs, total = lzr.compress(xd, p)
    torch.cuda.synchronize()
    tot = int(total.item())
    r_out, r_sizes, r_offs, r_tot = ref.compress(xd.cpu().numpy(), ref.Params(parse=1),
                                                 n_threads=len(os.sched_getaffinity(0)))
    assert tot == r_tot
    assert np.array_equal(sizes.cpu().numpy().view(np.uint32), r_sizes)
    assert np.array_equal(out[:tot].cpu().numpy(), r_out)
