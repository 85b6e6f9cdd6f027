"""The device build of the generators produces the same bytes as the host build (so the CUDA
path and the oracle see identical inputs at any size)."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from gen import pygen  # noqa: E402


@pytest.mark.parametrize("spec", [pygen.spec_wc(10_000, 1), pygen.spec_wc(1_000_000, 5),
                                  pygen.spec_sm(260_000, 2), pygen.spec_ii(4)], ids=["wc10k", "wc1m", "sm", "ii"])
def test_text_pages_identical(spec):
    h = pygen.host_text(spec, 3, page0=5)
    d = pygen.device_text(spec, 3, page0=5)
    assert np.array_equal(d["data"].cpu().numpy(), h["data"])
    assert np.array_equal(d["offsets"].cpu().numpy().view(np.uint64), h["offsets"])
    assert d["n"] == h["n"]


def test_km_points_identical():
    spec = pygen.KMSpec()
    h = pygen.host_km(spec, 100_003, i0=12345)
    d = pygen.device_km(spec, 100_003, i0=12345).cpu().numpy()
    assert np.array_equal(h.view(np.uint32), d.view(np.uint32))
