"""Test-side checkers, independent of both the oracle and the CUDA path.

* ``parse_stream``: reads a chunk's byte stream back into tokens under the
  flag-byte LZSS reading R1, written from the format description,
  not from either implementation.
* ``brute_tokens``: the greedy longest-then-nearest parse recomputed by brute
  force in a different formulation (full table of capped common-prefix lengths
  for every admissible distance, then argmax) -- only for tiny inputs.
* ``brute_tokens_lazy``: the one-step lazy parse (R21) from a
  precomputed table of best (length, distance) at every position, then a walk
  over the table -- a different formulation from the oracle's on-the-fly one.
* ``check_tokens``: properties every correct token stream satisfies.
"""
from __future__ import annotations


def parse_stream(s: bytes, n: int, m: int):
    """Tokens [(length, dist)] of a compressed (non-raw) chunk stream, or raise."""
    toks = []
    ip = 0
    produced = 0
    while produced < n:
        f = s[ip]
        ip += 1
        for bit in range(8):
            if produced == n:
                assert f >> bit == 0, "padding flag bits must be zero"
                break
            if (f >> bit) & 1:
                d = s[ip] | (s[ip + 1] << 8)
                ln = s[ip + 2] + m
                ip += 3
                toks.append((ln, d + 1))
                produced += ln
            else:
                ip += 1
                toks.append((1, 0))
                produced += 1
    assert ip == len(s), "stream has trailing bytes"
    assert produced == n
    return toks


def encoded_size(tokens) -> int:
    T = len(tokens)
    return (T + 7) // 8 + sum(1 if d == 0 else 3 for _, d in tokens)


def capped_lcp_table(x: bytes, p: int, W: int, M: int):
    """[(d, l(d))] for d = 1..min(W, p): capped common-prefix length (overlap allowed)."""
    n = len(x)
    cap = min(M, n - p)
    out = []
    for d in range(1, min(W, p) + 1):
        l = 0
        # compare against the ORIGINAL bytes (= byte-serial copy semantics)
        while l < cap and x[p + l] == x[p - d + l]:
            l += 1
        out.append((d, l))
    return out


def brute_tokens(x: bytes, W: int, m: int, M: int):
    n = len(x)
    p = 0
    toks = []
    while p < n:
        tab = capped_lcp_table(x, p, W, M)
        best = max((l for _, l in tab), default=0)
        if best >= m:
            d = min(d for d, l in tab if l == best)
            toks.append((best, d))
            p += best
        else:
            toks.append((1, 0))
            p += 1
    return toks


def best_table(x: bytes, W: int, M: int):
    """[(l*, d*)] at every position: longest capped match, smallest d among equals."""
    out = []
    for p in range(len(x)):
        tab = capped_lcp_table(x, p, W, M)
        best = max((l for _, l in tab), default=0)
        d = min((d for d, l in tab if l == best), default=0) if best else 0
        out.append((best, d))
    return out


def brute_tokens_lazy(x: bytes, W: int, m: int, M: int):
    n = len(x)
    bt = best_table(x, W, M)
    p = 0
    toks = []
    while p < n:
        l, d = bt[p]
        deferred = p + 1 < n and bt[p + 1][0] > l
        if l >= m and not deferred:
            toks.append((l, d))
            p += l
        else:
            toks.append((1, 0))
            p += 1
    return toks


def decode_tokens(x_literals_from: bytes, tokens) -> bytes:
    """Rebuild the chunk from tokens, taking literal bytes from the original."""
    out = bytearray()
    for ln, d in tokens:
        if d == 0:
            out.append(x_literals_from[len(out)])
        else:
            assert 1 <= d <= len(out)
            for _ in range(ln):
                out.append(out[-d])
    return bytes(out)


def check_tokens(x: bytes, tokens, W: int, m: int, M: int):
    n = len(x)
    assert sum(l for l, _ in tokens) == n
    p = 0
    for ln, d in tokens:
        if d:
            assert 1 <= d <= min(W, p)
            assert m <= ln <= min(M, n - p)
            for k in range(ln):
                assert x[p + k] == x[p - d + k]
        else:
            assert ln == 1
        p += ln
    assert decode_tokens(x, tokens) == x
