import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
# WordCount tables: libbmr counts exact / mid / long words in tables for every input size; below
# 64 MiB (BMR_XTAB_MIN_BYTES) without the 4 GiB direct-address exact-key table ("small-table mode":
# exact words that miss the SMEM combiner go to the mid table).  The small test inputs therefore
# run the small-table mode; tests/test_gpu_tables.py re-runs the WordCount cases with the exact-key
# table (BMR_XTAB_MIN_BYTES=0, the C5 path), and test_wc_small_input_sort_path the sorted streams.
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
