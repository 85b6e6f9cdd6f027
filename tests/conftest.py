import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
# the WordCount L2 count tables are used for every input size in the tests (libbmr's default skips
# them below 64 MiB, where sorting the exact keys is cheaper than streaming the table);
# test_wc_small_input_sort_path covers the other side
os.environ.setdefault("BMR_TABLE_MIN_BYTES", "0")
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a); run with -m gpu")


@pytest.fixture(scope="session", autouse=True)
def _built():
    """Make sure the native artefacts exist (build() is cheap when up to date)."""
    import __graft_entry__ as ge
    ge.build(quiet=True)
