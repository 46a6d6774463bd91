"""Pins of the dedup oracle (oracle/dedup_ref.c, oracle.dedup_index) against
what fixes it from outside: the published SHA-1 example digests (FIPS 180-2
Appendix A / FIPS 180-4 examples), Python's hashlib on random messages of every
length around the padding boundaries, and a brute-force first-occurrence
definition of the index (§2 "Indexing is the process of comparing the hash
value of each chunk with the hash values of already stored chunks").  CPU only."""
import hashlib
import json
import os

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _golden():
    with open(os.path.join(ROOT, "tests", "golden", "sha1_vectors.jsonl")) as f:
        return [json.loads(l) for l in f if l.strip()]


@pytest.mark.parametrize("vec", _golden(), ids=lambda v: v["name"])
def test_sha1_published_vectors(ref, vec):
    msg = vec["message"].encode() * vec.get("repeat", 1)
    assert ref.sha1(msg).hex() == vec["sha1"]


def test_sha1_every_length_vs_hashlib(ref):
    rng = np.random.default_rng(7)
    for n in range(0, 300):  # crosses the 55/56/63/64-byte padding cases several times
        x = rng.integers(0, 256, n, dtype=np.uint8).tobytes()
        assert ref.sha1(x) == hashlib.sha1(x).digest(), n


def test_fingerprints_vs_hashlib(ref):
    rng = np.random.default_rng(8)
    for C, n in [(4096, 5 * 4096), (4096, 3 * 4096 + 1000), (64, 64 * 7 + 63), (100, 1000), (1, 5)]:
        x = rng.integers(0, 256, n, dtype=np.uint8)
        fp = ref.fingerprints(x, C, n_threads=3)
        N = -(-n // C)
        assert fp.shape == (N, 20)
        for i in range(N):
            assert bytes(fp[i]) == hashlib.sha1(x[i * C:(i + 1) * C].tobytes()).digest()


def test_fingerprints_thread_invariance(ref):
    import synth

    x = synth.fill_host(64 * 4096, 4096, "mix")
    a = ref.fingerprints(x, 4096, n_threads=1)
    b = ref.fingerprints(x, 4096, n_threads=7)
    assert np.array_equal(a, b)


def _brute_index(fps, first=0):
    N = len(fps)
    idx = np.zeros(N, np.uint64)
    for i in range(N):
        j = next(j for j in range(i + 1) if bytes(fps[j]) == bytes(fps[i]))
        idx[i] = first + j
    return idx


def test_index_vs_brute_force(ref):
    rng = np.random.default_rng(9)
    for trial in range(30):
        N = int(rng.integers(1, 60))
        distinct = rng.integers(0, 256, (int(rng.integers(1, N + 1)), 20), dtype=np.uint8)
        fps = distinct[rng.integers(0, len(distinct), N)]
        first = int(rng.integers(0, 1000))
        idx, hit, _ = ref.dedup_index(fps, first)
        assert np.array_equal(idx, _brute_index(fps, first))
        assert np.array_equal(hit.astype(bool), idx != first + np.arange(N, dtype=np.uint64))


def test_index_batches_equal_whole(ref):
    rng = np.random.default_rng(10)
    distinct = rng.integers(0, 256, (40, 20), dtype=np.uint8)
    fps = distinct[rng.integers(0, 40, 200)]
    whole, _, _ = ref.dedup_index(fps, 0)
    seen = {}
    parts = []
    for lo in range(0, 200, 37):
        idx, _, seen = ref.dedup_index(fps[lo:lo + 37], lo, seen)
        parts.append(idx)
    assert np.array_equal(np.concatenate(parts), whole)


def test_dedup_stream_generator():
    """Config-5 stream (synth SYN_DEDUP): duplicates carry earlier fresh content,
    and the logical/unique ratio is ~2.0 (§4 "deduplication ... ratio are
    set to 2.0")."""
    import synth

    N = 4000
    src = np.array([synth.dedup_source(i) for i in range(N)])
    assert src[0] == 0 and np.all(src <= np.arange(N))
    assert np.all(src[src] == src)  # a source is fresh (its own source)
    ratio = N / len(np.unique(src))
    assert 1.85 < ratio < 2.15, ratio
    x = synth.fill_host(256 * 4096, 4096, "mix_dedup").reshape(256, 4096)
    base = synth.fill_host(256 * 4096, 4096, "mix").reshape(256, 4096)
    for i in range(256):
        assert np.array_equal(x[i], base[src[i]])
