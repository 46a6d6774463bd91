"""Pins for the fast exact CPU compressor (cpuref/)
against the plain oracle and the brute-force checker (-m "not gpu").

cpuref finds longest matches through hash chains and a run-aware search, so
its result must equal the oracle's exhaustive definition byte for byte:
every stream class, the adversarial inputs of the GPU parity tests (runs,
periods, small alphabets, ragged tails), a (C, W, m, M) grid incl. W < C, m = 3
and C = 32 KiB, both parse rules, and brute force on tiny inputs."""
import itertools
import random

import numpy as np
import pytest

import cpuref
import synth
from tests import lzss_check as lc
from tests.test_gpu_parity import _adversarial


def _same(ref, x, **kw):
    a = cpuref.compress(x, cpuref.Params(**kw), n_threads=4)
    b = ref.compress(x, ref.Params(**kw))
    assert a[3] == b[3]
    assert np.array_equal(a[1], b[1]) and np.array_equal(a[2], b[2])
    assert np.array_equal(a[0], b[0])
    return a


@pytest.mark.parametrize("parse", [0, 1])
@pytest.mark.parametrize("cls", ["mix", "text", "random", "zeroruns", "cr2"])
def test_classes_equal_oracle(ref, cls, parse):
    _same(ref, synth.fill_host(1 << 20, 4096, cls, seed=31), parse=parse)


@pytest.mark.parametrize("parse", [0, 1])
@pytest.mark.parametrize("name,x", list(_adversarial()), ids=lambda v: v if isinstance(v, str) else "")
def test_adversarial_equal_oracle(ref, name, x, parse):
    _same(ref, x, parse=parse)


@pytest.mark.parametrize("C,W,m,M", [
    (4096, 4096, 3, 258), (4096, 4096, 5, 40), (4096, 4096, 3, 3), (4096, 4096, 9, 12),
    (4096, 1000, 4, 259), (4096, 1, 4, 259), (4096, 2, 3, 100), (4096, 33, 6, 261),
    (16, 16, 3, 258), (16, 5, 4, 259), (528, 300, 4, 20), (8192, 8192, 4, 259),
    (16384, 4096, 4, 259), (32768, 32768, 4, 259),
])
def test_param_grid_equal_oracle(ref, C, W, m, M):
    n = max(C * 3 + C // 3 + 1, 3000)
    x = synth.fill_host(n, C, "mix", seed=C + W + m + M)
    for parse in (0, 1):
        _same(ref, x, chunk_size=C, window=W, min_match=m, max_match=M, parse=parse)


def test_bruteforce_small(ref):
    rng = random.Random(0xFA57)
    for it in range(1500):
        n = rng.randint(1, 64)
        alpha = rng.choice([1, 2, 3, 256])
        x = bytes(rng.randrange(alpha) for _ in range(n))
        W = max(1, rng.choice([1, 2, 3, 5, 8, n]))
        m = rng.choice([3, 4, 5])
        M = m + rng.choice([0, 1, 3, 255])
        for parse, brute in ((0, lc.brute_tokens), (1, lc.brute_tokens_lazy)):
            out, sizes, _, _ = cpuref.compress(x, cpuref.Params(chunk_size=64, window=W, min_match=m,
                                                                max_match=M, parse=parse), n_threads=1)
            toks = brute(x, W, m, M)
            if int(sizes[0]) < n:
                assert lc.parse_stream(out.tobytes(), n, m) == toks, (x, W, m, M, parse)
            else:
                assert out.tobytes() == x and lc.encoded_size(toks) >= n


def test_all_binary_strings(ref):
    for n in range(1, 11):
        for tup in itertools.product(b"ab", repeat=n):
            x = bytes(tup)
            for parse in (0, 1):
                p = dict(chunk_size=16, window=16, min_match=3, max_match=6, parse=parse)
                a = cpuref.compress(x, cpuref.Params(**p), n_threads=1)
                assert a[0].tobytes() == ref.compress_chunk(x, ref.Params(**p)), (x, parse)


def test_validation():
    assert cpuref.validate(cpuref.Params()) == 0
    assert cpuref.validate(cpuref.Params(parse=2)) == -2
    assert cpuref.validate(cpuref.Params(tie_break=1)) == -2
    assert cpuref.validate(cpuref.Params(chunk_size=24)) == -1


def test_cpu_dedup_arm_equals_oracle_index(ref):
    """The CPU dedup arm of the integration options (hashlib SHA-1 + first
    occurrence) == the oracle's fingerprints + index (R17, R18), tail chunk included."""
    import cpuref
    import synth

    for n, C in [((1 << 20) + 777, 4096), (300 * 512, 512), (5, 4096)]:
        x = synth.fill_host(n, C, "mix_dedup", seed=n)
        idx, un = cpuref.dedup(x, C, 4)
        r_idx, r_hit, _ = ref.dedup_index(ref.fingerprints(x, C), 0)
        assert np.array_equal(idx.astype(np.uint64), r_idx)
        assert np.array_equal(un.astype(bool), r_hit == 0)
