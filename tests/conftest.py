import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: long-running (full BASELINE sizes)")


@pytest.fixture(scope="session", autouse=True)
def _built():
    """Compile the (CPU-side) generator and oracle once per session."""
    import datagen
    import oracle
    import __graft_entry__
    datagen.build()
    oracle.build()
    nat = __graft_entry__._native()
    nat.build()              # libxreduce.so (no-op when up to date)
    nat.build_devapi_test()  # tests/devapi/libxr_devapi_test.so
    yield
