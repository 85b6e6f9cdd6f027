import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a); run with -m gpu")


@pytest.fixture(scope="session", autouse=True)
def _built():
    """Make sure the native artefacts exist (build() is cheap when up to date)."""
    import __graft_entry__ as ge
    ge.build(quiet=True)
