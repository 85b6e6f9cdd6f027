"""WordCount table modes against the oracle: the exact-key table
(`BMR_XTAB_MIN_BYTES=0`: exact words that miss the SMEM combiner are REDs into the 2^30-entry
direct-address table — the C5 path) and the small-table mode (the default below 64 MiB: those
words go to the open-addressing mid table, whose 48-bit keys include the 30-bit exact ones), on
the same inputs: both must equal the oracle and each other."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from gen import pygen  # noqa: E402
from tests.helpers import make_records  # noqa: E402
from tests.test_gpu_parity import _wc_edge_records, same  # noqa: E402

MODES = {"exact-table": "0", "small-table": str(1 << 40)}


def _cases():
    g1 = pygen.host_text(pygen.spec_wc(10_000, 1), 1)
    g5 = pygen.host_text(pygen.spec_wc(1_000_000, 5), 3)
    e = make_records(_wc_edge_records(3))
    return {"c1": (g1["data"], g1["offsets"], g1["n"]), "v1m": (g5["data"], g5["offsets"], g5["n"]),
            "edges": (e[0], e[1], len(e[1]) - 1)}


@pytest.mark.parametrize("case", ["c1", "v1m", "edges"])
def test_wc_table_modes_agree(case, monkeypatch):
    b = [_cases()[case]]
    got = {}
    for mode, xm in MODES.items():
        monkeypatch.setenv("BMR_XTAB_MIN_BYTES", xm)
        got[mode], st = same("wc", b)
        assert st["pairs"] == 0 or case == "edges"     # (edges: words > 16 bytes are hashed pairs)
    assert got["exact-table"] == got["small-table"]


def test_wc_small_table_exact_words_grow(monkeypatch):
    # 300k distinct 5-symbol words (exact keys), three times each: most miss the per-CTA SMEM
    # combiner, so in small-table mode they fill the mid table past its first 2^18 slots -> the Map
    # flags it, the table grows and the batch is replayed; the CTA-end combiner flush also inserts
    monkeypatch.setenv("BMR_XTAB_MIN_BYTES", str(1 << 40))
    alpha = np.frombuffer(b"abcdefghijklmnopqrstuvwxyzABCDEFGHIJKLMNOPQRSTUVWXYZ0123456789", np.uint8)
    idx = np.arange(300_000)
    words = [bytes(alpha[[(i // 62 ** k) % 62 for k in range(5)]].tolist()) for i in idx.tolist()]
    recs = [b" ".join(words[i:i + 7]) for i in range(0, len(words), 7)] * 3
    data, off = make_records(recs)
    got, st = same("wc", [(data, off, len(recs))])
    assert len(got) == 300_000 and set(got.values()) == {3}
    assert st["replays"] >= 1
