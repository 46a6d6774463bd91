"""Host-side checks of the C ABI (no GPU needed): liblzr.so loads, exports every
symbol include/lzr.h declares, and its host-only entry points (validation,
sizing, status strings, host argument checks) behave as documented."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def lzr():
    from paper_conf_pact_map17_b200 import _build

    _build.build()
    import paper_conf_pact_map17_b200 as m

    return m


def _declared_symbols():
    src = open(os.path.join(ROOT, "include", "lzr.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(lzr_[a-z_0-9]+)\s*\(", src)))


def test_header_symbols_exported(lzr):
    declared = _declared_symbols()
    assert "lzr_compress_chunks" in declared and "lzr_decompress_chunks" in declared
    nm = subprocess.run(["nm", "-D", "--defined-only", lzr.LIB_PATH], capture_output=True,
                        text=True, check=True).stdout
    exported = set(re.findall(r"\s[TW]\s+(lzr_\w+)", nm))
    missing = [s for s in declared if s not in exported]
    assert not missing, missing
    assert sorted(lzr.EXPORTED_SYMBOLS) == declared
    for s in declared:
        getattr(lzr.lib(), s)


def test_library_is_sm100a(lzr):
    out = subprocess.run(["cuobjdump", "--list-elf", lzr.LIB_PATH], capture_output=True, text=True)
    assert "sm_100a" in out.stdout


def test_validate_matches_oracle_rules(lzr, ref):
    import itertools
    for C, W, m, M, tb in itertools.product([8, 16, 4096, 4100, 65536, 65552], [0, 1, 4096, 70000],
                                            [2, 3, 4, 255, 256], [3, 4, 259, 260, 510], [0, 1]):
        g = lzr.validate_params(lzr.Params(C, W, m, M, tb))
        r = ref.validate(ref.Params(C, W, m, M, tb))
        assert g == r, (C, W, m, M, tb, g, r)


def test_sizing(lzr):
    p = lzr.Params()
    assert lzr.num_chunks(0, p) == 0
    assert lzr.num_chunks(1, p) == 1
    assert lzr.num_chunks(4096, p) == 1
    assert lzr.num_chunks(4097, p) == 2
    assert lzr.compress_bound(12345, p) == 12345
    w1 = lzr.compress_workspace_bytes(1 << 20, p)
    w2 = lzr.compress_workspace_bytes(1 << 21, p)
    assert w1 >= (1 << 20) and w2 > w1 and w1 % 256 == 0
    bad = lzr.Params(chunk_size=10)
    assert lzr.num_chunks(100, bad) == 0 and lzr.compress_workspace_bytes(100, bad) == 0
    assert lzr.status_str(0) == "LZR_OK" and lzr.status_str(-5) == "LZR_ERR_CORRUPT"


def test_host_argument_errors(lzr):
    L = lzr.lib()
    p = lzr.Params()
    cp = ctypes.byref(p.c())
    # NULL input with n > 0, misaligned input, small workspace: rejected before any launch
    assert L.lzr_compress_chunks(None, 4096, cp, ctypes.c_void_p(256), 4096, ctypes.c_void_p(256),
                                 ctypes.c_void_p(256), None, ctypes.c_void_p(256), 1 << 20,
                                 None) == lzr.ERR_INVALID_ARG
    assert L.lzr_compress_chunks(ctypes.c_void_p(4097), 4096, cp, ctypes.c_void_p(256), 4096,
                                 ctypes.c_void_p(256), ctypes.c_void_p(256), None,
                                 ctypes.c_void_p(256), 1 << 20, None) == lzr.ERR_INVALID_ARG
    assert L.lzr_compress_chunks(ctypes.c_void_p(4096), 4096, cp, ctypes.c_void_p(256), 100,
                                 ctypes.c_void_p(256), ctypes.c_void_p(256), None,
                                 ctypes.c_void_p(256), 1 << 20, None) == lzr.ERR_CAPACITY
    assert L.lzr_compress_encode(ctypes.c_void_p(4096), 4096, cp, ctypes.c_void_p(256),
                                 ctypes.c_void_p(256), 16, None) == lzr.ERR_CAPACITY
    tb = lzr.Params(tie_break=1)
    assert L.lzr_compress_chunks(ctypes.c_void_p(4096), 4096, ctypes.byref(tb.c()),
                                 ctypes.c_void_p(256), 4096, ctypes.c_void_p(256),
                                 ctypes.c_void_p(256), None, ctypes.c_void_p(256), 1 << 20,
                                 None) == lzr.ERR_UNSUPPORTED
    # parse rule: greedy (0) and lazy (1) are valid, anything else is unsupported
    assert L.lzr_validate_params(ctypes.byref(lzr.Params(parse=lzr.PARSE_LAZY).c())) == lzr.OK
    assert L.lzr_validate_params(ctypes.byref(lzr.Params(parse=2).c())) == lzr.ERR_UNSUPPORTED
    # n == 0 is a no-op
    assert L.lzr_compress_encode(None, 0, cp, None, None, 0, None) == lzr.OK
    # host-buffer decompression: n == 0 no-op (error word cleared), NULL
    # buffers / a batch that is not a multiple of C rejected before any CUDA call
    err = ctypes.c_int32(7)
    assert L.lzr_decompress_host(None, None, None, 0, cp, None, ctypes.byref(err), 0, None, 0) == lzr.OK
    assert err.value == 0
    v = ctypes.c_void_p(256)
    assert L.lzr_decompress_host(None, v, v, 4096, cp, v, None, 0, v, 1 << 30) == lzr.ERR_INVALID_ARG
    assert L.lzr_decompress_host(v, v, v, 8192, cp, v, None, 4000, v, 1 << 30) == lzr.ERR_INVALID_ARG
    assert L.lzr_decompress_host_scratch_bytes(1 << 20, cp) > 2 * (1 << 20)
    assert L.lzr_decompress_host_scratch_bytes(0, cp) == 0


def test_no_gpu_fails_loudly(lzr):
    torch = pytest.importorskip("torch")
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    L = lzr.lib()
    p = lzr.Params()
    st = L.lzr_compress_encode(ctypes.c_void_p(4096), 4096, ctypes.byref(p.c()),
                               ctypes.c_void_p(256), ctypes.c_void_p(256), 1 << 20, None)
    assert st == lzr.ERR_CUDA
    with pytest.raises(Exception):
        lzr.compress(torch.zeros(4096, dtype=torch.uint8), p)  # CPU tensor: no CPU path


def test_decoder_float_mod_identity():
    """decode.cu's periodic copies take x mod d (x <= 32, 1 <= d < 32) as
    x - d * floor((x + 0.5) * rcp(d)) in IEEE single precision: exact for every pair."""
    import numpy as np

    for d in range(1, 32):
        rd = np.float32(1.0) / np.float32(d)
        for x in range(0, 33):
            q = int(np.float32(np.float32(x) + np.float32(0.5)) * rd)
            assert q == x // d, (x, d)
