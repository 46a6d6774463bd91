"""Full-size parity at BASELINE.json's configs 3, 4 and 5 in the launch
configuration bench.py times (one GPU): deterministic chunk samples against the
oracle, EVERY chunk against the fast exact CPU compressor (cpuref/, itself
pinned to the oracle by tests/test_cpuref.py), and properties that hold at any
size (offsets = exclusive scan of sizes, full GPU round trip; for the dedup
stream, every index number equals the generator's ground-truth source chunk and
its fingerprint matches)."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import cpuref  # noqa: E402
import synth  # noqa: E402


@pytest.fixture(scope="module")
def lzr():
    assert torch.cuda.is_available(), "gpu tests need a CUDA device"
    import __graft_entry__

    __graft_entry__.build()
    import paper_conf_pact_map17_b200 as m

    return m


def _full_stream_check(xd, C, out, sizes, offs, parse=0, batch=256 << 20):
    """Every chunk, batch by batch: sizes and the compacted bytes of the batch
    equal cpuref's (= the oracle's definition) exactly."""
    n = xd.numel()
    N = -(-n // C)
    g_sizes = sizes.cpu().numpy().view(np.uint32)
    g_offs = offs.cpu().numpy().view(np.uint64)
    per = max(1, batch // C)
    slots = np.empty(per * C, np.uint8)
    for i0 in range(0, N, per):
        i1 = min(N, i0 + per)
        xs = xd[i0 * C: min(n, i1 * C)].cpu().numpy()
        c_out, c_sizes, _, c_tot = cpuref.compress(xs, cpuref.Params(chunk_size=C, parse=parse), slots=slots)
        assert np.array_equal(g_sizes[i0:i1], c_sizes), i0
        lo = int(g_offs[i0])
        got = out[lo: lo + int(c_tot)].cpu().numpy()
        if not np.array_equal(got, c_out):
            bad = int(np.argmax(got != c_out))
            raise AssertionError(f"batch at chunk {i0}: first differing byte {bad}")


def _sampled_check(lzr, ref, xd, C, every, roundtrip=True, full=True):
    n = xd.numel()
    p = lzr.Params(chunk_size=C)
    out, sizes, offs, total = lzr.compress(xd, p)
    torch.cuda.synchronize()
    N = -(-n // C)
    idx = sorted(set(range(0, N, every)) | set(range(min(N, 64))) | set(range(max(0, N - 64), N)))
    g_sizes = sizes.cpu().numpy().view(np.uint32)
    g_offs = offs.cpu().numpy().view(np.uint64)
    xs = np.concatenate([xd[i * C:(i + 1) * C].cpu().numpy() for i in idx])
    # the sampled chunks, compressed by the oracle one by one
    r_streams, r_sizes = ref.compress_sampled(xs, ref.Params(chunk_size=C), list(range(len(idx))))
    for k, i in enumerate(idx):
        assert g_sizes[i] == r_sizes[k], i
        got = out[int(g_offs[i]): int(g_offs[i]) + int(g_sizes[i])].cpu().numpy().tobytes()
        assert got == r_streams[k], i
    assert g_offs[0] == 0 and np.array_equal(g_offs[1:], np.cumsum(g_sizes[:-1], dtype=np.uint64))
    assert int(total.item()) == int(g_sizes.sum(dtype=np.uint64))
    if full:
        _full_stream_check(xd, C, out, sizes, offs)
    if roundtrip:
        y, err = lzr.decompress(out, sizes, offs, n, p)
        torch.cuda.synchronize()
        assert int(err.item()) == 0 and torch.equal(y, xd)
        del y
    del out


@pytest.mark.parametrize("C", [4096, 8192, 16384, 32768, 65536])
def test_config3_1gib_sampled(lzr, ref, C):
    xd = torch.empty(1 << 30, dtype=torch.uint8, device="cuda")
    synth.fill_device(xd, C, "mix")
    _sampled_check(lzr, ref, xd, C, every=1024 if C >= 16384 else 256)


def test_config3_1gib_lazy_full_stream(lzr):
    """The lazy parse (R21) over the whole 1 GiB mix stream, every chunk."""
    xd = torch.empty(1 << 30, dtype=torch.uint8, device="cuda")
    synth.fill_device(xd, 4096, "mix")
    p = lzr.Params(parse=lzr.PARSE_LAZY)
    out, sizes, offs, total = lzr.compress(xd, p)
    torch.cuda.synchronize()
    _full_stream_check(xd, 4096, out, sizes, offs, parse=1)


def test_config4_16gib_sampled(lzr, ref):
    xd = torch.empty(16 << 30, dtype=torch.uint8, device="cuda")
    synth.fill_device(xd, 4096, "mix")
    _sampled_check(lzr, ref, xd, 4096, every=4096)
    del xd
    torch.cuda.empty_cache()


def test_config5_16gib_dedup_properties(lzr, ref):
    C = 4096
    n = 16 << 30
    N = n // C
    xd = torch.empty(n, dtype=torch.uint8, device="cuda")
    synth.fill_device(xd, C, "mix_dedup")
    fp = lzr.fingerprint(xd, C)
    index = lzr.DedupIndex.for_chunks(N)
    idx, uniq = index.index(fp, 0)
    torch.cuda.synchronize()
    assert int(index.overflow.item()) == 0
    g_idx = idx.cpu().numpy().view(np.uint64)
    g_un = uniq.cpu().numpy()
    assert np.all(g_idx <= np.arange(N, dtype=np.uint64))
    assert np.array_equal(g_un.astype(bool), g_idx == np.arange(N, dtype=np.uint64))
    ratio = N / int(g_un.sum())
    assert 1.95 < ratio < 2.05, ratio  # P:18 §4 "deduplication ... ratio are set to 2.0"
    rng = np.random.default_rng(11)
    sample = sorted(set(rng.integers(0, N, 2000).tolist()) | set(range(64)) | set(range(N - 64, N)))
    for i in sample:
        # ground truth of the generator: the first occurrence of chunk i's content
        assert int(g_idx[i]) == synth.dedup_source(i), i
    for i in sample[:300]:  # fingerprints of the pair, by the oracle
        j = int(g_idx[i])
        a = ref.sha1(xd[i * C:(i + 1) * C].cpu().numpy())
        assert bytes(fp[i].cpu().numpy()) == a
        assert ref.sha1(xd[j * C:(j + 1) * C].cpu().numpy()) == a
