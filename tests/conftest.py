import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA GPU (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: long-running (still CPU-only unless also marked gpu)")


def pytest_collection_modifyitems(config, items):
    # A `-m gpu` run must not silently pass on a box without a GPU: the gpu
    # tests assert on the device themselves (see tests/gpu_util.py).
    pass


@pytest.fixture(scope="session")
def ref():
    import oracle

    oracle.build()
    return oracle
