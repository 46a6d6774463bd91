"""Pins for the CPU oracle (-m "not gpu").

The paper prints no worked example, no ratio and no token format (SURVEY.md §0,
§8(c)), so every pin here is self-constructed from the readings in DESIGN.md
and chosen so that a plausible slip in oracle/lzr_ref.c fails one of them:

* hand-worked byte-exact examples (tests/golden/appendix_a.jsonl): format
  bytes, flag bit order, offset/length bias, overlap, cap-before-tie-break,
  nearest tie-break, window, raw fallback;
* closed forms: constant chunks, periodic chunks;
* brute force (tests/lzss_check.py, a different formulation) on every binary
  string up to length 10 and on random short strings over a (W, m, M) grid;
* properties: round trip, stream/format self-consistency, chunk independence,
  exclusive-scan offsets, decoder error detection.
"""
import itertools
import json
import os
import random

import numpy as np
import pytest

from tests import lzss_check as lc

GOLDEN = [os.path.join(os.path.dirname(__file__), "golden", f)
          for f in ("appendix_a.jsonl", "lazy_examples.jsonl")]


def _golden():
    out = []
    for path in GOLDEN:
        with open(path) as f:
            out += [json.loads(l) for l in f if l.strip()]
    return out


def _params(ref, d):
    return ref.Params(**d)


@pytest.mark.parametrize("case", _golden(), ids=lambda c: c["id"])
def test_golden_appendix_a(ref, case):
    p = _params(ref, case["params"])
    if "input_ascii" in case:
        x = case["input_ascii"].encode()
    else:
        b, n = case["input_fill"]
        x = bytes([b]) * n
    if "tokens" in case:
        assert ref.parse_chunk(x, p) == [tuple(t) for t in case["tokens"]]
    s = ref.compress_chunk(x, p)
    assert len(s) == case["size"]
    assert s.hex() == case["expected_hex"]
    assert (len(s) == len(x)) == case["raw"]
    st, y = ref.decompress_chunk(s, len(x), p)
    assert st == 0 and y == x


def _const_closed_form(n, m, M):
    # first byte literal; then q full-cap matches at d=1; remainder r:
    # a match if r >= m, else r literals (cap < m)
    q, r = divmod(n - 1, M)
    matches = q + (1 if r >= m else 0)
    literals = 1 + (r if 0 < r < m else 0)
    T = matches + literals
    S = (T + 7) // 8 + literals + 3 * matches
    return min(S, n) if S < n else n


@pytest.mark.parametrize("n,expect", [(4096, 52), (8192, 102), (16384, 202), (32768, 398), (65536, 795)])
def test_constant_chunk_sizes(ref, n, expect):
    p = ref.Params(chunk_size=n)
    s = ref.compress_chunk(bytes(n), p)
    assert len(s) == expect
    assert len(s) == _const_closed_form(n, 4, 259)


@pytest.mark.parametrize("m", [3, 4, 5, 9])
@pytest.mark.parametrize("dM", [0, 1, 3, 17, 255])
def test_constant_chunk_closed_form_grid(ref, m, dM):
    M = m + dM
    for n in [1, 2, 3, 4, 5, 7, 8, 15, 16, 17, 31, 64, 100, 259, 260, 261, 263, 1000, 4096]:
        C = max(16, ((n + 15) // 16) * 16)
        p = ref.Params(chunk_size=C, window=C, min_match=m, max_match=M)
        for b in (0x00, 0xA5):
            s = ref.compress_chunk(bytes([b]) * n, p)
            assert len(s) == _const_closed_form(n, m, M), (n, m, M)


def test_periodic_chunk(ref):
    # q distinct bytes repeated: q literals, then matches at d = q (nearest) each capped at M
    x = (b"vwxyz" * 1000)[:4096]
    p = ref.Params()
    toks = ref.parse_chunk(x, p)
    assert toks[:5] == [(1, 0)] * 5
    assert all(d == 5 for _, d in toks[5:])
    assert len(toks) == 21
    assert len(ref.compress_chunk(x, p)) == 56
    for q in [1, 2, 3, 7, 31, 64, 255]:
        x = bytes((i % q) + 1 for i in range(4096))
        toks = ref.parse_chunk(x, p)
        assert toks[:q] == [(1, 0)] * q
        assert all(d == q for _, d in toks[q:])
        assert all(l == 259 for l, _ in toks[q:-1])


def test_period_beyond_window_is_literal(ref):
    # period 40 with W = 32: no admissible distance ever matches
    x = bytes((i * 7) % 40 for i in range(400))
    p = ref.Params(chunk_size=400 - 400 % 16 + 16, window=32)
    assert all(d == 0 for _, d in ref.parse_chunk(x, p))


def test_random_chunk_is_raw(ref):
    rng = random.Random(7)
    while True:
        x = bytes(rng.getrandbits(8) for _ in range(4096))
        grams = [x[i:i + 4] for i in range(4093)]
        if len(set(grams)) == len(grams):
            break
    p = ref.Params()
    assert all(d == 0 for _, d in ref.parse_chunk(x, p))
    s = ref.compress_chunk(x, p)
    assert s == x  # 4096 literals need 4608 B >= 4096 -> raw (R9)


def _grid(n):
    for W in sorted({1, 2, 3, 5, max(1, n)}):
        for m in (3, 4):
            for M in (m, m + 1, m + 3, m + 255):
                yield W, m, M


def test_bruteforce_all_binary_strings(ref):
    # every string over {a,b} of length 1..10, small (W, m, M) grid
    checked = 0
    for n in range(1, 11):
        for tup in itertools.product(b"ab", repeat=n):
            x = bytes(tup)
            for W, m, M in _grid(n):
                if W > 16:
                    continue
                p = ref.Params(chunk_size=16, window=W, min_match=m, max_match=M)
                toks = ref.parse_chunk(x, p)
                assert toks == lc.brute_tokens(x, W, m, M), (x, W, m, M)
                checked += 1
    assert checked > 10000


def test_bruteforce_random_strings(ref):
    rng = random.Random(0x4C5A52)
    for it in range(3000):
        n = rng.randint(1, 64)
        alpha = rng.choice([2, 4, 256])
        x = bytes(rng.randrange(alpha) for _ in range(n))
        W = rng.choice([1, 2, 3, 5, 8, n])
        m = rng.choice([3, 4, 5])
        M = m + rng.choice([0, 1, 3, 255])
        p = ref.Params(chunk_size=64, window=max(1, W), min_match=m, max_match=M)
        toks = ref.parse_chunk(x, p)
        assert toks == lc.brute_tokens(x, max(1, W), m, M), (x, W, m, M)
        lc.check_tokens(x, toks, max(1, W), m, M)
        s = ref.compress_chunk(x, p)
        if len(s) < n:
            assert lc.parse_stream(s, n, m) == toks
            assert len(s) == lc.encoded_size(toks)
        else:
            assert s == x and lc.encoded_size(toks) >= n
        st, y = ref.decompress_chunk(s, n, p)
        assert st == 0 and y == x


# ---- one-step lazy parse (R21) -----------------

def test_lazy_bruteforce_all_binary_strings(ref):
    checked = differ = 0
    for n in range(1, 11):
        for tup in itertools.product(b"ab", repeat=n):
            x = bytes(tup)
            for W, m, M in _grid(n):
                if W > 16:
                    continue
                p = ref.Params(chunk_size=16, window=W, min_match=m, max_match=M, parse=1)
                toks = ref.parse_chunk(x, p)
                assert toks == lc.brute_tokens_lazy(x, W, m, M), (x, W, m, M)
                differ += toks != lc.brute_tokens(x, W, m, M)
                checked += 1
    assert checked > 10000 and differ > 100  # the two parses really differ


def test_lazy_bruteforce_random_strings(ref):
    rng = random.Random(0x1A2F)
    for it in range(2000):
        n = rng.randint(1, 64)
        alpha = rng.choice([2, 4, 256])
        x = bytes(rng.randrange(alpha) for _ in range(n))
        W = max(1, rng.choice([1, 2, 3, 5, 8, n]))
        m = rng.choice([3, 4, 5])
        M = m + rng.choice([0, 1, 3, 255])
        p = ref.Params(chunk_size=64, window=W, min_match=m, max_match=M, parse=1)
        toks = ref.parse_chunk(x, p)
        assert toks == lc.brute_tokens_lazy(x, W, m, M), (x, W, m, M)
        lc.check_tokens(x, toks, W, m, M)
        s = ref.compress_chunk(x, p)
        if len(s) < n:
            assert lc.parse_stream(s, n, m) == toks
        st, y = ref.decompress_chunk(s, n, p)
        assert st == 0 and y == x


def test_lazy_equals_greedy_on_constant_and_periodic(ref):
    # the best length never grows from p to p+1 on constant / periodic data
    # (it is min(M, n-p) once the first period is history), so nothing is
    # deferred: the closed forms of the greedy parse hold unchanged
    for n in (4096, 8192):
        p = ref.Params(chunk_size=n, parse=1)
        assert len(ref.compress_chunk(bytes(n), p)) == _const_closed_form(n, 4, 259)
    for q in [1, 2, 3, 5, 7, 31, 255]:
        x = bytes((i % q) + 1 for i in range(4096))
        assert ref.parse_chunk(x, ref.Params(parse=1)) == ref.parse_chunk(x, ref.Params())


def test_lazy_stream_roundtrip(ref):
    import synth
    x = synth.fill_host(64 * 4096, 4096, "mix", seed=5)
    p = ref.Params(parse=1)
    out, sizes, offsets, total = ref.compress(x, p)
    st, bad, y = ref.decompress(out, sizes, offsets, x.size, p)
    assert st == 0 and bad == 0 and np.array_equal(y, x)
    _, g_sizes, _, _ = ref.compress(x, ref.Params())
    assert not np.array_equal(sizes, g_sizes)  # lazy changes some chunks


def test_param_validation(ref):
    P = ref.Params
    assert ref.validate(P()) == 0
    assert ref.validate(P(chunk_size=8)) == ref.ERR_INVALID_ARG
    assert ref.validate(P(chunk_size=4100)) == ref.ERR_INVALID_ARG
    assert ref.validate(P(chunk_size=65536 + 16)) == ref.ERR_INVALID_ARG
    assert ref.validate(P(window=0)) == ref.ERR_INVALID_ARG
    assert ref.validate(P(window=4097)) == ref.ERR_INVALID_ARG
    assert ref.validate(P(min_match=2)) == ref.ERR_INVALID_ARG
    assert ref.validate(P(min_match=4, max_match=3)) == ref.ERR_INVALID_ARG
    assert ref.validate(P(min_match=4, max_match=260)) == ref.ERR_INVALID_ARG
    assert ref.validate(P(tie_break=1)) == ref.ERR_UNSUPPORTED
    assert ref.validate(P(parse=1)) == ref.OK
    assert ref.validate(P(parse=2)) == ref.ERR_UNSUPPORTED


def _mixed_stream(n, seed):
    rng = np.random.default_rng(seed)
    parts = []
    tot = 0
    while tot < n:
        k = int(rng.integers(0, 3))
        ln = int(rng.integers(8, 600))
        if k == 0:
            parts.append(np.zeros(ln, np.uint8))
        elif k == 1:
            parts.append(rng.integers(0, 256, ln, dtype=np.uint8))
        else:
            words = [b"alpha ", b"beta ", b"gamma ", b"delta, ", b"the ", b"of "]
            s = b"".join(words[int(i)] for i in rng.integers(0, len(words), ln // 4 + 1))
            parts.append(np.frombuffer(s[:ln], np.uint8))
        tot += ln
    return np.concatenate(parts)[:n].copy()


def test_stream_driver_offsets_independence_and_tail(ref):
    p = ref.Params(chunk_size=512)
    x = _mixed_stream(512 * 37 + 77, 3)  # ragged tail chunk of 77 B
    out, sizes, offs, total = ref.compress(x, p, n_threads=4)
    N = ref.num_chunks(x.size, p)
    assert N == 38 and sizes.size == N
    assert offs[0] == 0 and np.all(offs[1:] == np.cumsum(sizes[:-1].astype(np.uint64)))
    assert total == int(sizes.astype(np.uint64).sum()) == out.size
    for i in range(N):
        lo, hi = i * 512, min(x.size, (i + 1) * 512)
        alone = ref.compress_chunk(x[lo:hi], p)  # chunks are independent (§3.2(1))
        assert out[offs[i]: offs[i] + sizes[i]].tobytes() == alone
        assert sizes[i] <= hi - lo
    st, bad, y = ref.decompress(out, sizes, offs, x.size, p)
    assert st == 0 and bad == 0 and np.array_equal(x, y)
    # thread count does not change anything
    out1, sizes1, _, _ = ref.compress(x, p, n_threads=1)
    assert np.array_equal(out1, out) and np.array_equal(sizes1, sizes)
    # sampled == full
    idx = [0, 5, 36, 37]
    outs, ss = ref.compress_sampled(x, p, idx)
    for k, i in enumerate(idx):
        assert outs[k] == out[offs[i]: offs[i] + sizes[i]].tobytes()


def test_empty_stream(ref):
    out, sizes, offs, total = ref.compress(np.zeros(0, np.uint8), ref.Params())
    assert total == 0 and sizes.size == 0


def _corrupt_cases():
    # base: "abcabcabcabc" -> 08 61 62 63 02 00 05 (A.1), n = 12, m = 4
    good = bytes.fromhex("08616263020005")
    yield "ok", good, 0
    yield "truncated", good[:-1], -5
    yield "trailing", good + b"\x00", -5
    yield "dist_too_far", bytes.fromhex("08616263030005"), -5  # d = 4 > 3 produced
    yield "overrun", bytes.fromhex("08616263020006"), -5  # l = 10 > 9 left
    yield "pad_bits", bytes.fromhex("18616263020005"), -5  # bit 4 set after n reached
    yield "S>n", good + bytes(6), -5


@pytest.mark.parametrize("name,s,expect", list(_corrupt_cases()), ids=lambda v: v if isinstance(v, str) else "")
def test_decoder_errors(ref, name, s, expect):
    p = ref.Params()
    st, y = ref.decompress_chunk(s, 12, p)
    assert st == expect
    if expect == 0:
        assert y == b"abcabcabcabc"


def test_decoder_reports_first_bad_chunk(ref):
    p = ref.Params(chunk_size=16)
    x = np.frombuffer(b"abcabcabcabcabca" * 3, np.uint8).copy()
    out, sizes, offs, total = ref.compress(x, p)
    bad_out = out.copy()
    bad_out[offs[1] + sizes[1] - 3] = 0xFF  # chunk 1: make d too far
    st, bad, _ = ref.decompress(bad_out, sizes, offs, x.size, p)
    assert st == ref.ERR_CORRUPT and bad == 2
