"""GPU parity of the dedup step through the C ABI against
the CPU oracle: SHA-1 fingerprints byte for byte, the index numbers and
hit/miss flags exactly (first occurrence in stream order, across batches),
the gather of unique chunks, and dedup-before-compression end to end (the
compressed unique stream bit-exact with the oracle's compression of the
oracle's unique chunks, plus a round trip back to the logical stream)."""
import hashlib

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


def _fp(lzr, x, C):
    xd = torch.from_numpy(np.ascontiguousarray(x)).cuda()
    fp = lzr.fingerprint(xd, C)
    torch.cuda.synchronize()
    return fp.cpu().numpy()


@pytest.mark.parametrize("C,n", [(4096, 300 * 4096), (4096, 37 * 4096 + 1234), (8192, 50 * 8192),
                                 (64, 64 * 1000 + 5), (100, 100 * 333 + 55), (1, 77), (4096, 10)])
def test_fingerprints_match_oracle(lzr, ref, C, n):
    x = synth.fill_host(n, C if C >= 16 else 16, "mix") if n >= 16 else np.arange(n, dtype=np.uint8)
    g = _fp(lzr, x, C)
    r = ref.fingerprints(x, C)
    assert g.shape == r.shape
    assert np.array_equal(g, r)


def test_fingerprint_unaligned_input(lzr, ref):
    x = synth.fill_host(20 * 4096 + 8, 4096, "text")
    xd = torch.from_numpy(x).cuda()[3:]  # 3-byte offset: byte-load path
    fp = lzr.fingerprint(xd, 4096)
    torch.cuda.synchronize()
    assert np.array_equal(fp.cpu().numpy(), ref.fingerprints(x[3:], 4096))


def test_fingerprint_empty(lzr):
    fp = lzr.fingerprint(torch.empty(0, dtype=torch.uint8, device="cuda"), 4096)
    assert fp.shape[0] == 0


def _index_check(lzr, ref, fps, batches, n_bins, slots):
    idx = lzr.DedupIndex(n_bins, slots)
    fpd = torch.from_numpy(np.ascontiguousarray(fps)).cuda()
    seen = {}
    g_all, u_all, r_all, h_all = [], [], [], []
    lo = 0
    for b in batches:
        gi, gu = idx.index(fpd[lo:lo + b], lo)
        torch.cuda.synchronize()
        ri, rh, seen = ref.dedup_index(fps[lo:lo + b], lo, seen)
        g_all.append(gi.cpu().numpy().view(np.uint64))
        u_all.append(gu.cpu().numpy())
        r_all.append(ri)
        h_all.append(rh)
        lo += b
    assert int(idx.overflow.item()) == 0
    g, u, r, h = map(np.concatenate, (g_all, u_all, r_all, h_all))
    assert np.array_equal(g, r)
    assert np.array_equal(u.astype(bool), ~h.astype(bool))


def test_index_matches_oracle_dedup_stream(lzr, ref):
    C = 4096
    x = synth.fill_host(3000 * C, C, "mix_dedup")
    fps = ref.fingerprints(x, C)
    _index_check(lzr, ref, fps, [3000], 256, 32)
    _index_check(lzr, ref, fps, [1, 999, 1000, 1000], 97, 64)  # batches, odd bin count


def test_index_heavy_duplicates_and_collisions(lzr, ref):
    rng = np.random.default_rng(3)
    distinct = rng.integers(0, 256, (50, 20), dtype=np.uint8)
    distinct[:10, :8] = distinct[0, :8]  # same bin and start slot, different fingerprints
    fps = distinct[rng.integers(0, 50, 20000)]
    _index_check(lzr, ref, fps, [20000], 4, 32)
    _index_check(lzr, ref, fps, [7000, 13000], 1, 128)


def test_index_overflow_is_reported(lzr):
    rng = np.random.default_rng(4)
    fps = torch.from_numpy(rng.integers(0, 256, (100, 20), dtype=np.uint8)).cuda()
    idx = lzr.DedupIndex(1, 16)
    gi, gu = idx.index(fps, 0)
    torch.cuda.synchronize()
    assert int(idx.overflow.item()) == 100 - 16
    assert int(gu.sum().item()) == 100  # not found => reported new


def test_gather_and_dedup_compress_end_to_end(lzr, ref):
    C = 4096
    n = 2000 * C + 777  # ragged tail chunk
    x = synth.fill_host(n, C, "mix_dedup")
    xd = torch.from_numpy(x).cuda()
    p = lzr.Params()
    res = lzr.dedup_compress(xd, p)
    torch.cuda.synchronize()
    # oracle: fingerprints -> first-occurrence index -> unique chunks in order
    fps = ref.fingerprints(x, C)
    ri, rh, _ = ref.dedup_index(fps, 0)
    N = fps.shape[0]
    uniq = np.flatnonzero(rh == 0)
    assert np.array_equal(res["index"].cpu().numpy().view(np.uint64), ri)
    assert res["n_unique"] == len(uniq)
    ub = np.concatenate([x[i * C:(i + 1) * C] for i in uniq])
    assert np.array_equal(res["unique_bytes"].cpu().numpy(), ub)
    r_out, r_sizes, r_offs, r_tot = ref.compress(ub, ref.Params())
    tot = int(res["total"].item())
    assert tot == r_tot
    assert np.array_equal(res["sizes"].cpu().numpy().view(np.uint32), r_sizes)
    assert np.array_equal(res["out"][:tot].cpu().numpy(), r_out)
    # restore the logical stream: decode the unique chunks, then copy each
    # duplicate from its index number's chunk
    y, err = lzr.decompress(res["out"], res["sizes"], res["offsets"], ub.size, p)
    torch.cuda.synchronize()
    assert int(err.item()) == 0
    yu = y.cpu().numpy()
    rank = {int(c): k for k, c in enumerate(uniq)}
    for i in range(N):
        src = rank[int(ri[i])]
        got = yu[src * C:src * C + min(C, n - i * C)]
        assert np.array_equal(got, x[i * C:(i + 1) * C]), i
    assert hashlib.sha1(x[:C].tobytes()).digest() == bytes(res["fp"][0].cpu().numpy())
