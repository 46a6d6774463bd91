"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle,
byte for byte (0-byte tolerance on output bytes, sizes and offsets; integer
work, so bit-exact is the bar -- DESIGN.md §Parity).

Sizes span several warps/CTAs and ragged tails; the full-size config-2 case
checks a deterministic chunk sample against the oracle plus a full GPU round
trip, in the launch configuration bench.py times.
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

pytestmark = pytest.mark.gpu

import synth  # noqa: E402


@pytest.fixture(scope="module")
def lzr():
    assert torch.cuda.is_available(), "gpu tests need a CUDA device"
    import __graft_entry__

    __graft_entry__.build()
    import paper_conf_pact_map17_b200 as m

    return m


def _ref_params(ref, p):
    return ref.Params(chunk_size=p.chunk_size, window=p.window, min_match=p.min_match,
                      max_match=p.max_match, parse=p.parse)


def _gpu_compress(lzr, x: np.ndarray, p):
    xd = torch.from_numpy(np.ascontiguousarray(x)).cuda()
    out, sizes, offs, total = lzr.compress(xd, p)
    torch.cuda.synchronize()
    tot = int(total.item())
    return (xd, out, sizes, offs, tot,
            out[:tot].cpu().numpy(), sizes.cpu().numpy().view(np.uint32),
            offs.cpu().numpy().view(np.uint64))


def _check_full(lzr, ref, x: np.ndarray, p, roundtrip=True):
    xd, out, sizes, offs, tot, g_out, g_sizes, g_offs = _gpu_compress(lzr, x, p)
    r_out, r_sizes, r_offs, r_tot = ref.compress(x, _ref_params(ref, p))
    assert tot == r_tot
    assert np.array_equal(g_sizes, r_sizes)
    assert np.array_equal(g_offs, r_offs)
    if not np.array_equal(g_out, r_out):
        bad = int(np.argmax(g_out != r_out))
        ci = int(np.searchsorted(r_offs, bad, side="right") - 1)
        raise AssertionError(f"first differing byte {bad} in chunk {ci}")
    if roundtrip:
        y, err = lzr.decompress(out, sizes, offs, x.size, p)
        torch.cuda.synchronize()
        assert int(err.item()) == 0
        assert torch.equal(y, xd)
    return g_out, g_sizes, g_offs


def test_config1_mix_bitexact(lzr, ref):
    x = synth.fill_host(1 << 20, 4096, "mix")
    _check_full(lzr, ref, x, lzr.Params())


@pytest.mark.parametrize("cls", ["text", "random", "zeroruns", "cr2"])
def test_classes_bitexact(lzr, ref, cls):
    x = synth.fill_host(1 << 20, 4096, cls, seed=11)
    _check_full(lzr, ref, x, lzr.Params())


def _adversarial():
    rng = np.random.default_rng(5)
    yield "zeros", np.zeros(4096 * 9, np.uint8)
    yield "ones_ragged", np.full(4096 * 3 + 5, 0xFF, np.uint8)
    yield "random_ragged", rng.integers(0, 256, 4096 * 5 + 1234, dtype=np.uint8)
    for q in [1, 2, 3, 4, 5, 7, 8, 16, 31, 32, 33, 63, 64, 200]:
        base = rng.integers(0, 256, q, dtype=np.uint8)
        yield f"period{q}", np.tile(base, 4096 * 2 // q + 2)[: 4096 * 2 + 77]
    yield "binary", rng.integers(0, 2, 4096 * 6, dtype=np.uint8)
    yield "quaternary", rng.integers(0, 4, 4096 * 6, dtype=np.uint8) + 0x61
    yield "runs", np.repeat(rng.integers(0, 3, 4000, dtype=np.uint8), rng.integers(1, 40, 4000))[: 4096 * 8]
    # run structure (exercises the run-aware search and its >64-runs fallback)
    vals = rng.integers(0, 3, 3000, dtype=np.uint8)
    lens = rng.integers(1, 300, 3000)
    yield "runs_long_3vals", np.repeat(vals, lens)[: 4096 * 8 + 100]
    yield "runs_short_many", np.repeat(rng.integers(0, 2, 6000, dtype=np.uint8), rng.integers(3, 9, 6000))[: 4096 * 6]
    zr = []
    for k in range(400):
        zr.append(np.zeros(int(rng.integers(4, 600)), np.uint8))
        zr.append(rng.integers(0, 256, int(rng.integers(1, 20)), dtype=np.uint8))
    yield "zero_runs_mixed_tails", np.concatenate(zr)[: 4096 * 10 + 7]
    pat = []
    for k in range(600):  # runs followed by repeated tails: exact-RL candidates with continuations
        pat.append(np.full(int(rng.integers(4, 40)), int(rng.integers(0, 2)), np.uint8))
        pat.append(np.frombuffer(b"xyz" if k % 3 else b"xyw", np.uint8))
    yield "runs_with_shared_tails", np.concatenate(pat)[: 4096 * 6]
    yield "tiny1", np.array([7], np.uint8)
    yield "tiny5", np.frombuffer(b"aaaaa", np.uint8).copy()


@pytest.mark.parametrize("name,x", list(_adversarial()), ids=lambda v: v if isinstance(v, str) else "")
def test_adversarial_bitexact(lzr, ref, name, x):
    _check_full(lzr, ref, x, lzr.Params())


@pytest.mark.parametrize("C,W,m,M", [
    (4096, 4096, 3, 258), (4096, 4096, 5, 40), (4096, 4096, 3, 3), (4096, 4096, 9, 12), (4096, 4096, 4, 4), (4096, 4096, 4, 5),
    (4096, 1000, 4, 259), (4096, 1, 4, 259), (4096, 2, 3, 100), (4096, 33, 6, 261),
    (16, 16, 3, 258), (16, 5, 4, 259), (48, 48, 4, 259), (528, 300, 4, 20),
    (8192, 8192, 4, 259), (16384, 16384, 4, 259), (32768, 32768, 4, 259),
    # big chunks (C > 32 KiB): 16-bit positions, bucket ends,
    # in-bucket search for p's entry, walk bitmaps in global scratch
    (65536, 65536, 4, 259), (65536, 65536, 3, 258), (65536, 20000, 4, 259), (40000, 40000, 4, 259),
    (32784, 32784, 5, 100),
    # 16-warp groups (8 KiB < C <= 32 KiB), incl. sizes that are not powers of two
    (8208, 8000, 3, 200), (12288, 12288, 4, 259), (24576, 1000, 4, 259),
])
def test_param_grid_bitexact(lzr, ref, C, W, m, M):
    p = lzr.Params(chunk_size=C, window=W, min_match=m, max_match=M)
    n = max(C * 3 + C // 3 + 1, 3000)
    x = synth.fill_host(n, C, "mix", seed=C + W + m + M)
    _check_full(lzr, ref, x, p)


@pytest.mark.parametrize("nchunks", [1, 2, 31, 32, 33, 147, 148, 149, 11 * 148 - 1, 11 * 148 + 1])
def test_batch_edges(lzr, ref, nchunks):
    x = synth.fill_host(nchunks * 4096, 4096, "mix", seed=nchunks)
    _check_full(lzr, ref, x, lzr.Params(), roundtrip=True)


def test_golden_through_gpu(lzr, ref):
    import json, os
    lines = []
    for f in ("appendix_a.jsonl", "lazy_examples.jsonl"):
        lines += open(os.path.join(os.path.dirname(__file__), "golden", f)).readlines()
    for line in lines:
        c = json.loads(line)
        pp = c["params"]
        p = lzr.Params(chunk_size=pp["chunk_size"], window=pp["window"], min_match=pp["min_match"],
                       max_match=pp["max_match"], parse=pp.get("parse", 0))
        if "input_ascii" in c:
            x = np.frombuffer(c["input_ascii"].encode(), np.uint8).copy()
        else:
            x = np.full(c["input_fill"][1], c["input_fill"][0], np.uint8)
        _, _, _, _, tot, g_out, g_sizes, _ = _gpu_compress(lzr, x, p)
        assert tot == c["size"] and g_out.tobytes().hex() == c["expected_hex"], c["id"]


def test_config2_full_size_sampled(lzr, ref):
    """256 MiB mix at the bench's launch configuration: deterministic sample
    (every 256th chunk + first/last 64) vs the oracle, full round trip."""
    n = 256 << 20
    p = lzr.Params()
    xd = torch.empty(n, dtype=torch.uint8, device="cuda")
    synth.fill_device(xd, 4096, "mix")
    x = xd.cpu().numpy()
    assert np.array_equal(x[: 1 << 20], synth.fill_host(1 << 20, 4096, "mix"))  # host == device gen
    out, sizes, offs, total = lzr.compress(xd, p)
    torch.cuda.synchronize()
    N = n // 4096
    idx = sorted(set(range(0, N, 256)) | set(range(64)) | set(range(N - 64, N)))
    g_sizes = sizes.cpu().numpy().view(np.uint32)
    g_offs = offs.cpu().numpy().view(np.uint64)
    g_out = out.cpu().numpy()
    r_streams, r_sizes = ref.compress_sampled(x, _ref_params(ref, p), idx)
    for k, i in enumerate(idx):
        assert g_sizes[i] == r_sizes[k], i
        assert g_out[g_offs[i]: g_offs[i] + g_sizes[i]].tobytes() == r_streams[k], i
    assert g_offs[0] == 0 and np.array_equal(g_offs[1:], np.cumsum(g_sizes[:-1], dtype=np.uint64))
    assert int(total.item()) == int(g_sizes.sum(dtype=np.uint64))
    y, err = lzr.decompress(out, sizes, offs, n, p)
    torch.cuda.synchronize()
    assert int(err.item()) == 0 and torch.equal(y, xd)


def test_config2_full_size_every_chunk_vs_oracle(lzr, ref):
    """All 65,536 chunks of the bench's 256 MiB mix stream vs the oracle itself
    (thread per chunk on the host cores, ~20 s on 16): sizes, offsets, total
    and every byte (full-size parity not only through cpuref)."""
    import os

    n = 256 << 20
    p = lzr.Params()
    xd = torch.empty(n, dtype=torch.uint8, device="cuda")
    synth.fill_device(xd, 4096, "mix")
    out, sizes, offs, total = lzr.compress(xd, p)
    torch.cuda.synchronize()
    tot = int(total.item())
    r_out, r_sizes, r_offs, r_tot = ref.compress(xd.cpu().numpy(), _ref_params(ref, p),
                                                 n_threads=len(os.sched_getaffinity(0)))
    assert tot == r_tot
    assert np.array_equal(sizes.cpu().numpy().view(np.uint32), r_sizes)
    assert np.array_equal(offs.cpu().numpy().view(np.uint64), r_offs)
    assert np.array_equal(out[:tot].cpu().numpy(), r_out)


def test_cross_decode_with_oracle(lzr, ref):
    x = synth.fill_host(3 << 20, 4096, "cr2", seed=99)
    g_out, g_sizes, g_offs = _check_full(lzr, ref, x, lzr.Params(), roundtrip=False)
    st, bad, y = ref.decompress(g_out, g_sizes, g_offs, x.size, ref.Params())
    assert st == 0 and np.array_equal(y, x)


def test_gpu_decoder_matches_oracle_on_corruption(lzr, ref):
    x = synth.fill_host(64 * 4096, 4096, "text", seed=3)
    p = lzr.Params()
    xd, out, sizes, offs, tot, g_out, g_sizes, g_offs = _gpu_compress(lzr, x, p)
    rng = np.random.default_rng(1)
    for trial in range(40):
        bad = g_out.copy()
        bs = g_sizes.copy()
        kind = trial % 3
        ci = int(rng.integers(0, 64))
        if g_sizes[ci] == 4096:
            continue
        if kind == 0:  # flip a random byte inside chunk ci
            pos = int(g_offs[ci] + rng.integers(0, g_sizes[ci]))
            bad[pos] ^= np.uint8(1 << int(rng.integers(0, 8)))
        elif kind == 1:  # truncate chunk ci by one byte
            bs[ci] -= 1
        else:  # claim one more byte
            bs[ci] += 1 if bs[ci] + 1 < 4096 else 0
        st, r_bad, _ = ref.decompress(bad, bs, g_offs, x.size, ref.Params())
        d_bad = torch.from_numpy(bad).cuda()
        d_bs = torch.from_numpy(bs.view(np.int32)).cuda()
        _, err = lzr.decompress(d_bad, d_bs, offs, x.size, p)
        torch.cuda.synchronize()
        assert int(err.item()) == r_bad, (trial, kind, ci)


def test_scan_sizes_large(lzr):
    rng = np.random.default_rng(2)
    for n in [1, 7, 2048, 2049, 100003, 5_000_000]:
        s = rng.integers(0, 4097, n, dtype=np.uint32)
        d = torch.from_numpy(s.view(np.int32)).cuda()
        offs, tot = lzr.scan_sizes(d, base=12345)
        torch.cuda.synchronize()
        exp = np.concatenate([[0], np.cumsum(s[:-1], dtype=np.uint64)]) + np.uint64(12345)
        assert np.array_equal(offs.cpu().numpy().view(np.uint64), exp)
        assert int(tot.item()) == 12345 + int(s.sum(dtype=np.uint64))


@pytest.mark.parametrize("n", [(8 << 20) + 4096 * 3 + 100, 8 << 20])
def test_compress_host_pipeline(lzr, ref, n):
    # (a ragged last chunk and an exact multiple of the batch size)
    x = synth.fill_host(n, 4096, "mix", seed=21)
    h = torch.from_numpy(x).pin_memory()
    for batch in [0, 1 << 20, 3 * 4096 * 128]:
        h_out, h_sizes, h_offs, tot = lzr.compress_host(h, lzr.Params(), batch_bytes=batch)
        xd, out, sizes, offs, dtot, g_out, g_sizes, g_offs = _gpu_compress(lzr, x, lzr.Params())
        assert tot == dtot
        assert np.array_equal(h_sizes.numpy().view(np.uint32), g_sizes)
        assert np.array_equal(h_offs.numpy().view(np.uint64), g_offs)
        assert np.array_equal(h_out[:tot].numpy(), g_out)


@pytest.mark.parametrize("C", [16384, 32768, 65536])
def test_compress_host_pipeline_large_chunks(lzr, ref, C):
    """The host pipeline with 16- and 32-warp groups (walk bitmaps in the L2
    scratch of every batch's workspace) == the device path == the oracle."""
    n = C * 13 + 4112
    x = synth.fill_host(n, C, "mix", seed=C)
    p = lzr.Params(chunk_size=C)
    h = torch.from_numpy(x).pin_memory()
    h_out, h_sizes, h_offs, tot = lzr.compress_host(h, p, batch_bytes=4 * C)
    r_out, r_sizes, r_offs, r_tot = ref.compress(x, _ref_params(ref, p))
    assert tot == r_tot
    assert np.array_equal(h_sizes.numpy().view(np.uint32), r_sizes)
    assert np.array_equal(h_offs.numpy().view(np.uint64), r_offs)
    assert np.array_equal(h_out[:tot].numpy(), r_out)


@pytest.mark.parametrize("C,batch", [(4096, 0), (4096, 1 << 20), (4096, 3 * 4096 * 7), (16384, 4 * 16384),
                                     (65536, 2 * 65536)])
def test_decompress_host_pipeline(lzr, ref, C, batch):
    """lzr_decompress_host (H2D of each batch's streams, decode, D2H) inverts
    lzr_compress_host, ragged tail included; a corrupted stream is reported at
    the same chunk as the oracle's decoder reports it."""
    n = C * 37 + 1000
    x = synth.fill_host(n, C, "mix", seed=C + batch)
    p = lzr.Params(chunk_size=C)
    h = torch.from_numpy(x).pin_memory()
    h_out, h_sizes, h_offs, tot = lzr.compress_host(h, p, batch_bytes=1 << 20)
    y, err = lzr.decompress_host(h_out, h_sizes, h_offs, n, p, batch_bytes=batch)
    assert err == 0 and np.array_equal(y.numpy(), x)
    # corrupt one compressed (non-raw) chunk in a later batch: same verdict as the oracle
    sz = h_sizes.numpy().view(np.uint32)
    nonraw = [i for i in range(sz.size) if sz[i] < min(C, n - i * C)]
    i = nonraw[len(nonraw) // 2]
    bad = h_out.clone()
    o = int(h_offs.numpy().view(np.uint64)[i])
    bad[o] ^= 0xFF  # the first flag byte: token kinds change
    r_st, r_bad, _ = ref.decompress(bad.numpy()[: int(tot)], sz, h_offs.numpy().view(np.uint64), n,
                                    ref.Params(chunk_size=C))
    _, err2 = lzr.decompress_host(bad, h_sizes, h_offs, n, p, batch_bytes=batch)
    assert err2 == r_bad


def test_empty_input(lzr):
    xd = torch.empty(0, dtype=torch.uint8, device="cuda")
    out, sizes, offs, total = lzr.compress(xd, lzr.Params())
    torch.cuda.synchronize()
    assert sizes.numel() == 0 and int(total.item()) == 0


@pytest.mark.timeout(300)
@pytest.mark.parametrize("C", [4096, 8192])
def test_repeated_launch_stress(lzr, C):
    """Many back-to-back launches on one workspace (a lane-divergent progress read
    once split warps in the speculative walk and deadlocked a warp-sync; this
    exercises the meeting logic under varying timing).  Results must be stable."""
    p = lzr.Params(chunk_size=C)
    n = 256 << 20
    xd = torch.empty(n, dtype=torch.uint8, device="cuda")
    synth.fill_device(xd, C, "mix", seed=C)
    ws = lzr.Workspace(n, p, xd.device)
    ref_total = None
    for i in range(12):
        out, sizes, offs, total = lzr.compress(xd, p, ws=ws)
        torch.cuda.synchronize()
        t = int(total.item())
        ref_total = t if ref_total is None else ref_total
        assert t == ref_total
    y, err = lzr.decompress(out, sizes, offs, n, p)
    torch.cuda.synchronize()
    assert int(err.item()) == 0 and torch.equal(y, xd)


def _mutate(rng, s: bytes, n: int) -> bytes:
    """One random corruption (or a random valid-looking edit) of a chunk stream."""
    b = bytearray(s)
    kind = int(rng.integers(0, 7))
    if kind == 0 and b:  # flip a bit
        i = int(rng.integers(0, len(b)))
        b[i] ^= 1 << int(rng.integers(0, 8))
    elif kind == 1 and b:  # a flag byte (the first) to a random value
        b[0] = int(rng.integers(0, 256))
    elif kind == 2 and len(b) > 1:  # truncate
        b = b[: int(rng.integers(0, len(b)))]
    elif kind == 3:  # trailing garbage
        b += bytes(rng.integers(0, 256, int(rng.integers(1, 4)), dtype=np.uint8))
    elif kind == 4:  # random stream of random length (< n: not raw)
        b = bytearray(rng.integers(0, 256, int(rng.integers(1, n)), dtype=np.uint8))
    elif kind == 5 and len(b) > 3:  # a length / distance byte to an extreme
        i = int(rng.integers(1, len(b)))
        b[i] = 0xFF if rng.integers(0, 2) else 0x00
    else:  # all flags set in the first group
        if b:
            b[0] = 0xFF
    if len(b) >= n:  # keep it a "compressed" chunk (size == n means raw)
        b = b[: n - 1]
    return bytes(b)


@pytest.mark.parametrize("C,m,cls", [(4096, 4, "text"), (4096, 4, "zeroruns"), (1024, 3, "cr2"),
                                     (256, 9, "text")])
def test_gpu_decoder_fuzz_vs_oracle(lzr, ref, C, m, cls):
    """Random corruptions of 1-3 chunks per trial: the GPU decoder's verdict
    (first bad chunk) equals the oracle decoder's; when every chunk is still
    valid, the outputs are equal byte for byte."""
    nch = 24
    x = synth.fill_host(nch * C - 77, C, cls, seed=C + m)
    p = lzr.Params(chunk_size=C, min_match=m)
    rp = _ref_params(ref, p)
    _, _, _, _, _, g_out, g_sizes, g_offs = _gpu_compress(lzr, x, p)
    streams = [g_out[g_offs[i]: g_offs[i] + g_sizes[i]].tobytes() for i in range(g_sizes.size)]
    ns = [min(C, x.size - i * C) for i in range(g_sizes.size)]
    comp_ok = [i for i in range(len(streams)) if g_sizes[i] < ns[i]]
    assert comp_ok, "need compressed chunks"
    rng = np.random.default_rng(C * 31 + m)
    n_valid = 0
    for trial in range(60):
        ss = list(streams)
        for ci in rng.choice(comp_ok, size=int(rng.integers(1, 4)), replace=False):
            ss[int(ci)] = _mutate(rng, ss[int(ci)], ns[int(ci)])
        sizes = np.array([len(s) for s in ss], np.uint32)
        offs = np.concatenate([[0], np.cumsum(sizes[:-1], dtype=np.uint64)]).astype(np.uint64)
        comp = np.frombuffer(b"".join(ss) + b"\0", np.uint8)
        st, r_bad, r_y = ref.decompress(comp, sizes, offs, x.size, rp)
        y, err = lzr.decompress(torch.from_numpy(comp.copy()).cuda(),
                                torch.from_numpy(sizes.view(np.int32)).cuda(),
                                torch.from_numpy(offs.view(np.int64)).cuda(), x.size, p)
        torch.cuda.synchronize()
        assert int(err.item()) == r_bad, (trial, r_bad)
        if r_bad == 0:
            n_valid += 1
            assert np.array_equal(y.cpu().numpy(), r_y), trial


@pytest.mark.parametrize("C,W,m", [(4096, 4096, 3), (4096, 4096, 5), (8192, 8192, 4), (32768, 32768, 4),
                                   (4096, 4095, 4), (4096, 4094, 4), (8192, 8192, 3),
                                   (65536, 65536, 4), (65536, 65536, 3), (65536, 65535, 4)])
def test_runs_structures_param_grid(lzr, ref, C, W, m):
    """Run-heavy chunks across m, C and W around the 'every prefix in the window'
    boundary: the index leaves repeated-byte keys out (run-aware search only) iff
    the runs fit the run list and W + 1 >= n; both sides of that switch must give
    the oracle's bytes."""
    rng = np.random.default_rng(C + W + m)
    parts = []
    for k in range(3000):
        parts.append(np.full(int(rng.integers(1, 70)), int(rng.integers(0, 4)), np.uint8))
        if k % 5 == 0:
            parts.append(rng.integers(0, 256, int(rng.integers(1, 12)), dtype=np.uint8))
    x = np.concatenate(parts)[: C * 4 + 333]
    _check_full(lzr, ref, x, lzr.Params(chunk_size=C, window=W, min_match=m))
    z = synth.fill_host(C * 6, C, "zeroruns", seed=m)
    _check_full(lzr, ref, z, lzr.Params(chunk_size=C, window=W, min_match=m))


def test_compress_host_concurrent_callers(lzr, ref):
    """Three host threads in lzr_compress_host at once on one device: the first
    takes the device's cached streams, the others private sets (capi.cu
    HostStreams); every result equals the device path's, greedy and lazy."""
    import threading

    jobs = []
    for t, (cls, parse) in enumerate([("mix", 0), ("text", 1), ("zeroruns", 0)]):
        x = synth.fill_host((4 << 20) + 4096 * t + 77, 4096, cls, seed=40 + t)
        jobs.append((x, lzr.Params(parse=parse)))
    res = [None] * len(jobs)

    def run(i):
        x, p = jobs[i]
        h = torch.from_numpy(x).pin_memory()
        for _ in range(3):
            res[i] = lzr.compress_host(h, p, batch_bytes=1 << 20)

    ths = [threading.Thread(target=run, args=(i,)) for i in range(len(jobs))]
    for th in ths:
        th.start()
    for th in ths:
        th.join()
    for (x, p), (h_out, h_sizes, h_offs, tot) in zip(jobs, res):
        _, _, _, _, dtot, g_out, g_sizes, g_offs = _gpu_compress(lzr, x, p)
        assert tot == dtot
        assert np.array_equal(h_sizes.numpy().view(np.uint32), g_sizes)
        assert np.array_equal(h_offs.numpy().view(np.uint64), g_offs)
        assert np.array_equal(h_out[:tot].numpy(), g_out)


def test_decode_without_error_word(lzr):
    """d_error == NULL through the C ABI: the stream still decodes (nothing is
    reported; the library keeps no error word of its own, include/lzr.h)."""
    import ctypes

    x = synth.fill_host(1 << 20, 4096, "mix", seed=3)
    p = lzr.Params()
    xd = torch.from_numpy(x).cuda()
    out, sizes, offs, total = lzr.compress(xd, p)
    y = torch.empty_like(xd)
    st = lzr.lib().lzr_decompress_chunks(
        lzr._ptr(out), lzr._ptr(sizes), lzr._ptr(offs), x.size, ctypes.byref(p.c()), lzr._ptr(y),
        ctypes.c_void_p(0), ctypes.c_void_p(0), 0, ctypes.c_void_p(torch.cuda.current_stream().cuda_stream))
    assert st == 0
    torch.cuda.synchronize()
    assert torch.equal(y, xd)


def test_other_stream_dedup_and_compress(lzr, ref):
    """dedup_compress / compress on a non-default stream size their
    buffers from values produced on that stream (no stale host reads)."""
    x = synth.fill_host(4 << 20, 4096, "mix_dedup", seed=5)
    xd = torch.from_numpy(x).cuda()
    s = torch.cuda.Stream()
    p = lzr.Params()
    for _ in range(3):
        res = lzr.dedup_compress(xd, p, stream=s)
        s.synchronize()
        r_idx, r_hit, _ = ref.dedup_index(ref.fingerprints(x, 4096), 0)
        assert res["n_unique"] == int((r_hit == 0).sum())
        ub = np.concatenate([x[i * 4096:(i + 1) * 4096] for i in np.flatnonzero(r_hit == 0)])
        r_out, _, _, r_tot = ref.compress(ub, ref.Params())
        assert int(res["total"].item()) == r_tot
        assert np.array_equal(res["out"][:r_tot].cpu().numpy(), r_out)


@pytest.mark.parametrize("cls", ["text", "zeroruns", "random", "cr2"])
def test_big_chunk_classes_bitexact(lzr, ref, cls):
    """C = W = 64 KiB (the format's largest window, d - 1 < 2^16) on every class,
    plus a whole-chunk zero run (run end = 65536) and a period-3 chunk."""
    C = 65536
    x = synth.fill_host(C * 3 + 4112, C, cls, seed=64)
    _check_full(lzr, ref, x, lzr.Params(chunk_size=C))


def test_big_chunk_edge_inputs(lzr, ref):
    C = 65536
    _check_full(lzr, ref, np.zeros(C * 2, np.uint8), lzr.Params(chunk_size=C))
    per = np.tile(np.frombuffer(b"xyz", np.uint8), C // 3 + 1)[: C + 77].copy()
    _check_full(lzr, ref, per, lzr.Params(chunk_size=C))
    rng = np.random.default_rng(9)
    words = [bytes(rng.integers(97, 123, int(rng.integers(3, 9)), dtype=np.uint8)) for _ in range(40)]
    t = b" ".join(words[int(i)] for i in rng.integers(0, 40, 30000))[: C * 2 - 5]
    _check_full(lzr, ref, np.frombuffer(t, np.uint8).copy(), lzr.Params(chunk_size=C))


@pytest.mark.parametrize("seed", range(32))
def test_random_params_fuzz(lzr, ref, seed):
    """Seeded random (C, W, m, M, parse, class) configurations across every
    kernel family (1..32 warps per chunk, the big layout) vs the oracle."""
    rng = np.random.default_rng(1000 + seed)
    C = int(rng.choice([16, 48, 512, 1024, 2064, 4096, 6144, 8192, 12288, 16384, 20480, 32768, 49152, 65536]))
    W = int(rng.integers(1, C + 1)) if rng.random() < 0.5 else C
    m = int(rng.integers(3, 8))
    M = m + int(rng.integers(0, 256))
    parse = int(rng.integers(0, 2))
    cls = str(rng.choice(["mix", "text", "zeroruns", "cr2"]))
    n = int(C * rng.integers(2, 5) + rng.integers(0, C))
    x = synth.fill_host(n, C, cls, seed=seed)
    _check_full(lzr, ref, x, lzr.Params(chunk_size=C, window=W, min_match=m, max_match=M, parse=parse))


def _decoder_paths_inputs(C: int, m: int, seed: int):
    """Chunks built to drive the decoder's step paths (decode.cu): (A) all-match
    streams of (m + 1)-byte copies from the first quarter -- groups of 25 bytes, so a
    step takes 5 of its 8 groups, and more than 32 final-sourced matches per
    step (list overflow into the token-order pass); (B) periodic runs with
    periods 1..70 (overlapping matches, d < l, both below and above 32);
    (C) words from a small vocabulary (short matches reading the same step's
    output: the token-order pass)."""
    rng = np.random.default_rng(seed)
    q = C // 4
    a = []
    for _ in range(3):
        head = rng.integers(0, 256, q, dtype=np.uint8)
        offs = rng.integers(0, q - m - 1, (C - q) // (m + 1) + 1)
        a.append(np.concatenate([head, np.concatenate([head[o:o + m + 1] for o in offs])])[:C])
    b = []
    for _ in range(3):
        parts, tot = [], 0
        while tot < C:
            per = int(rng.integers(1, 71))
            ln = int(rng.integers(per + 1, per + 300))
            base = rng.integers(0, 256, per, dtype=np.uint8)
            parts.append(np.tile(base, ln // per + 1)[:ln])
            tot += ln
        b.append(np.concatenate(parts)[:C])
    vocab = [rng.integers(97, 123, int(rng.integers(3, 8)), dtype=np.uint8) for _ in range(16)]
    c = []
    for _ in range(3):
        parts, tot = [], 0
        while tot < C:
            w = vocab[int(rng.integers(0, 16))]
            parts.append(np.append(w, np.uint8(32)))
            tot += w.size + 1
        c.append(np.concatenate(parts)[:C])
    return np.concatenate(a + b + c + [c[0][: C // 3]])  # + a ragged tail chunk


@pytest.mark.parametrize("C,m", [(4096, 4), (4096, 3), (1024, 3), (4096, 6), (65536, 4)])
def test_decoder_step_paths_vs_oracle(lzr, ref, C, m):
    """GPU decode of oracle-compressed streams (the two share no code) that
    drive the decoder's step paths; the first kind must really put > 32 match
    tokens into one 64-token step."""
    from tests.lzss_check import parse_stream

    x = _decoder_paths_inputs(C, m, seed=C + m)
    rp = ref.Params(chunk_size=C, window=C, min_match=m, max_match=m + 255)
    r_out, r_sizes, r_offs, r_tot = ref.compress(x, rp)
    if C <= 4096:
        toks = parse_stream(bytes(r_out[r_offs[1]:r_offs[1] + r_sizes[1]]), C, m)
        assert max(sum(1 for ln, d in toks[i:i + 64] if d) for i in range(0, len(toks), 64)) > 32
    p = lzr.Params(chunk_size=C, min_match=m)
    d_out = torch.from_numpy(r_out).cuda()
    d_sizes = torch.from_numpy(r_sizes.view(np.int32)).cuda()
    d_offs = torch.from_numpy(r_offs.view(np.int64)).cuda()
    for sched in (True, False):  # costliest-first schedule and index order
        y, err = lzr.decompress(d_out, d_sizes, d_offs, x.size, p, schedule=sched)
        torch.cuda.synchronize()
        assert int(err.item()) == 0
        assert np.array_equal(y.cpu().numpy(), x)


def test_decode_schedule_workspace_and_order(lzr, ref):
    """The decode schedule: too small a workspace is LZR_ERR_CAPACITY; with and
    without a workspace the output and the first-corrupt-chunk verdict agree
    (the schedule changes the order chunks are decoded in, not the result)."""
    import ctypes

    x = synth.fill_host(64 * 4096 + 999, 4096, "mix", seed=21)
    p = lzr.Params()
    xd, out, sizes, offs, tot, g_out, g_sizes, g_offs = _gpu_compress(lzr, x, p)
    need = lzr.lib().lzr_decompress_workspace_bytes(x.size, ctypes.byref(p.c()))
    assert need >= 4 * (128 + 65)
    small = torch.empty(need - 4, dtype=torch.uint8, device="cuda")
    with pytest.raises(lzr.LzrError):
        lzr.decompress(out, sizes, offs, x.size, p, workspace=small)
    for sched in (True, False):
        y, err = lzr.decompress(out, sizes, offs, x.size, p, schedule=sched)
        torch.cuda.synchronize()
        assert int(err.item()) == 0 and torch.equal(y, xd)
    # two corrupt chunks: the lower index is reported whichever is decoded first
    bad = g_out.copy()
    for ci in (40, 9):
        if g_sizes[ci] < 4096:
            bad[g_offs[ci] + 1] ^= 0xFF
    st, r_bad, _ = ref.decompress(bad, g_sizes, g_offs, x.size, ref.Params())
    d_bad = torch.from_numpy(bad).cuda()
    for sched in (True, False):
        _, err = lzr.decompress(d_bad, sizes, offs, x.size, p, schedule=sched)
        torch.cuda.synchronize()
        assert int(err.item()) == r_bad
