"""Integration-option selection (§4(3)): every
placement of dedup and compression (GPU / CPU / split) gives the oracle's
result -- index numbers, unique flags (R17/R18) and the compressed unique
stream (R1-R9) -- and the placement the dummy-I/O calibration picks does too."""
import os

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def integ():
    assert torch.cuda.is_available()
    import __graft_entry__
    __graft_entry__.build()
    import cpuref
    import paper_conf_pact_map17_b200 as lzr
    from paper_conf_pact_map17_b200.integration import CpuArm, Integrated

    cores = len(os.sched_getaffinity(0))
    arm = CpuArm(compress=lambda x, p: cpuref.compress(x, cpuref.Params(chunk_size=p.chunk_size, window=p.window,
                                                                         parse=p.parse), n_threads=cores),
                 dedup=lambda x, C: cpuref.dedup(x, C, cores), cores=cores)
    return lzr, Integrated, arm


def _oracle_result(ref, x, C, parse=0):
    idx, hit, _ = ref.dedup_index(ref.fingerprints(x, C), 0)
    keep = np.flatnonzero(hit == 0)
    ub = np.concatenate([x[i * C:(i + 1) * C] for i in keep]) if keep.size else np.zeros(0, np.uint8)
    out, sizes, offs, tot = ref.compress(ub, ref.Params(chunk_size=C, parse=parse))
    return idx, (hit == 0).astype(np.int32), out, sizes, offs, tot


def _same(r, o):
    idx, un, out, sizes, offs, tot = o
    assert np.array_equal(r["index"].astype(np.uint64), idx)
    assert np.array_equal(r["unique"], un)
    assert r["total"] == tot
    assert np.array_equal(r["sizes"], sizes)
    assert np.array_equal(r["offsets"], offs)
    assert np.array_equal(r["out"], out)


@pytest.mark.parametrize("placement", ["gpu_both", "gpu_dedup_cpu_compress", "cpu_dedup_gpu_compress",
                                       "cpu_both", "gpu_dedup_split"])
@pytest.mark.parametrize("n,tail", [(4 << 20, 0), (1 << 20, 777)])
def test_every_placement_equals_oracle(integ, ref, placement, n, tail):
    lzr, Integrated, arm = integ
    import synth

    C = 4096
    x = synth.fill_host(n + tail, C, "mix_dedup", seed=21)
    it = Integrated(lzr.Params(), arm, "cuda", split_fraction=0.3)
    _same(it.run(x, placement), _oracle_result(ref, x, C))


def test_calibration_pick_equals_oracle(integ, ref):
    lzr, Integrated, arm = integ
    import synth

    C = 4096
    it = Integrated(lzr.Params(), arm, "cuda")
    cal = it.calibrate(synth.fill_host(16 << 20, C, "mix_dedup", seed=2), repeats=1)
    assert set(cal["gbs"]) == {"gpu_both", "gpu_dedup_cpu_compress", "cpu_dedup_gpu_compress", "cpu_both",
                               "gpu_dedup_split"}
    assert cal["pick"] == max(cal["gbs"], key=cal["gbs"].get)
    assert 0.0 <= cal["split_fraction"] < 1.0
    x = synth.fill_host(8 << 20, C, "mix_dedup", seed=23)
    _same(it.run(x, cal["pick"]), _oracle_result(ref, x, C))
    _same(it.run(x, "gpu_dedup_split"), _oracle_result(ref, x, C))
