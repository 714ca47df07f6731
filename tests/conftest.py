import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (sm_100a) GPU; runs the CUDA path through the C-ABI")
    config.addinivalue_line("markers", "slow: long CPU test (oracle at larger sizes)")


@pytest.fixture(scope="session", autouse=True)
def _built():
    """Make sure the native artefacts exist (gcc/nvcc builds are incremental)."""
    import __graft_entry__

    __graft_entry__.build()
