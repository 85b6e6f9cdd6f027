"""Pins for the CPU oracle (oracle/) against things other than itself (task rule ③):
brute force in plain Python, generator ground truth, closed forms, invariants, special
cases and the paper's worked example.  CPU only."""
import re
from collections import Counter

import numpy as np
import pytest

from gen import pygen
from oracle import oracle
from tests.helpers import decode, make_records, split_records

WORD = re.compile(rb"[0-9A-Za-z]+")


def brute_wc(recs):
    c = Counter()
    for r in recs:
        c.update(WORD.findall(r))
    return dict(c)


def rand_records(rng, n, maxlen=40, alphabet=b"ab AB09,.\n\x80\xffz"):
    return [bytes(rng.choice(list(alphabet), size=rng.integers(0, maxlen + 1)).tolist()) for _ in range(n)]


# ---------------- WordCount ----------------
@pytest.mark.parametrize("seed", range(6))
def test_wc_bruteforce_tiny(seed):
    rng = np.random.default_rng(seed)
    recs = rand_records(rng, int(rng.integers(0, 60)))
    data, off = make_records(recs)
    r = oracle.run("wc", [(data, off, len(recs), 0, 0)])
    assert decode("wc", r) == brute_wc(recs)


def test_wc_words_never_span_records():
    recs = [b"ab", b"cd", b"", b"e f", b"gh"]
    data, off = make_records(recs)
    r = decode("wc", oracle.run("wc", [(data, off, len(recs), 0, 0)]))
    assert r == {b"ab": 1, b"cd": 1, b"e": 1, b"f": 1, b"gh": 1}


def test_wc_fig2_golden():
    lines = open("tests/golden/fig2_wc.txt").read().splitlines()
    recs = [bytes.fromhex(h) for h in next(l for l in lines if l.startswith("records:")).split()[1:]]
    exp = [t.split(":") for t in next(l for l in lines if l.startswith("expect:")).split()[1:]]
    data, off = make_records(recs)
    assert [len(x) for x in recs] == [2, 3, 2]
    r = decode("wc", oracle.run("wc", [(data, off, 3, 0, 0)]))
    assert r == {w.encode(): 1 for w, _ in exp}
    assert [len(w) for w, _ in exp] == [int(s) for _, s in exp] == [1, 3, 2]


def test_wc_generator_ground_truth_c1():
    spec = pygen.spec_wc(10_000, 1)
    g = pygen.host_text(spec, 1, truth=True)
    r = oracle.run("wc", [(g["data"], g["offsets"], g["n"], 0, 0)])
    got = decode("wc", r)
    hist = g["word_hist"]
    exp = {pygen.word(i): int(c) for i, c in enumerate(hist) if c}
    assert got == exp
    assert sum(got.values()) == int(hist.sum()) == r["pairs"]          # Σcounts = tokens
    # ~200k words per MiB and ~10k vocab (BASELINE configs[0])
    assert 150_000 < r["pairs"] < 250_000
    assert 5_000 < len(got) <= 10_000


def test_wc_vocab_one_special_case():
    spec = pygen.spec_wc(1, 1)
    g = pygen.host_text(spec, 1, truth=True)
    got = decode("wc", oracle.run("wc", [(g["data"], g["offsets"], g["n"], 0, 0)]))
    assert got == {pygen.word(0): int(g["word_hist"][0])}


def test_wc_multibatch_equals_single():
    spec = pygen.spec_wc(1000, 11)
    g = pygen.host_text(spec, 2)
    data, off = g["data"], g["offsets"]
    cut = int(g["n"] // 3)
    b0 = (data[: int(off[cut])], off[: cut + 1], cut, 0, 0)
    b1 = (data[int(off[cut]):], off[cut:] - off[cut], g["n"] - cut, 0, int(off[cut]))
    one = oracle.run("wc", [(data, off, g["n"], 0, 0)])
    two = oracle.run("wc", [b0, b1])
    assert decode("wc", one) == decode("wc", two)


# ---------------- StringMatch ----------------
def brute_sm(recs, pat, base_offsets):
    out = []
    for r, b in zip(recs, base_offsets):
        for j in range(0, len(r) - 15):
            if r[j:j + 16] == pat:
                out.append(b + j)
    return np.array(sorted(out), np.uint64)


@pytest.mark.parametrize("seed", range(4))
def test_sm_bruteforce_tiny(seed):
    rng = np.random.default_rng(100 + seed)
    pat = b"abababababababab"
    recs = []
    for _ in range(40):
        r = bytearray(rng.choice(list(b"ab "), size=int(rng.integers(0, 60))).tolist())
        if rng.random() < 0.5 and len(r) >= 16:
            j = int(rng.integers(0, len(r) - 15))
            r[j:j + 16] = pat
        recs.append(bytes(r))
    data, off = make_records(recs)
    base = 1000
    got = decode("sm", oracle.run("sm", [(data, off, len(recs), 0, base)], pattern=pat))
    exp = brute_sm(recs, pat, [base + int(o) for o in off[:-1]])
    assert np.array_equal(got, exp)


@pytest.mark.parametrize("seed", range(4))
def test_sm_lines_bruteforce(seed):
    # the paper's per-line StringMatch (L125: "emit the line if found"): Python `in` per record
    rng = np.random.default_rng(300 + seed)
    pat = b"abababababababab"
    recs = []
    for _ in range(60):
        r = bytearray(rng.choice(list(b"ab "), size=int(rng.integers(0, 70))).tolist())
        for _ in range(int(rng.integers(0, 3))):
            if len(r) >= 16:
                j = int(rng.integers(0, len(r) - 15))
                r[j:j + 16] = pat
        recs.append(bytes(r))
    data, off = make_records(recs)
    base = 77
    got = decode("sm", oracle.run("sml", [(data, off, len(recs), 0, base)], pattern=pat))
    exp = np.array([base + int(off[i]) for i, r in enumerate(recs) if pat in r], np.uint64)
    assert np.array_equal(got, exp) and len(exp) > 0
    # every line of the per-offset output's records, once
    per_off = decode("sm", oracle.run("sm", [(data, off, len(recs), 0, base)], pattern=pat))
    starts = np.array([base + int(o) for o in off[:-1]], np.uint64)
    rec_of = np.searchsorted(starts, per_off, side="right") - 1
    assert np.array_equal(np.unique(starts[rec_of]), got)


def test_sm_self_overlap_985():
    data, off = make_records([b"a" * 1000])
    got = decode("sm", oracle.run("sm", [(data, off, 1, 0, 0)], pattern=b"a" * 16))
    assert len(got) == 985 and np.array_equal(got, np.arange(985, dtype=np.uint64))


def test_sm_no_match_across_records():
    pat = b"0123456789abcdef"
    data, off = make_records([b"xx0123456789", b"abcdefyy", pat])
    got = decode("sm", oracle.run("sm", [(data, off, 3, 0, 0)], pattern=pat))
    assert got.tolist() == [20]


def test_sm_planted_set_equals_found_set():
    spec = pygen.spec_sm(plant_ppm=20_000, cid=2)
    g = pygen.host_text(spec, 8, truth=True)
    got = decode("sm", oracle.run("sm", [(g["data"], g["offsets"], g["n"], 0, 0)], pattern=spec.pattern))
    assert len(g["plants"]) > 1000
    assert np.array_equal(got, g["plants"])
    b = bytes(g["data"])
    for o in got[:50]:
        assert b[int(o):int(o) + 16] == spec.pattern


# ---------------- KMeans ----------------
def _quantised(rng, n, k):
    pts = (rng.integers(-60_000, 60_000, size=(n, 8)) / 1024.0).astype(np.float32)
    cen = (rng.integers(-60_000, 60_000, size=(k, 8)) / 1024.0).astype(np.float32)
    return pts, cen


@pytest.mark.parametrize("seed", range(3))
def test_km_assignment_vs_exact_distances(seed):
    """The fp32 fmaf rule may differ from the exact argmin only within 2^-21 relative (C-4)."""
    rng = np.random.default_rng(seed)
    pts, cen = _quantised(rng, 3000, 7)
    r = oracle.run("km", [(pts.view(np.uint8).reshape(-1), None, len(pts), 32, 0)], centroids=cen)
    c_new, cnt = decode("km", r)
    # recover the oracle's assignment from counts + means is not possible; use exact distances:
    d = ((pts.astype(np.float64)[:, None, :] - cen.astype(np.float64)[None]) ** 2).sum(-1)
    best = d.min(1)
    # every point's assigned cluster (the one reproducing the oracle means) must be near-optimal:
    exact = d.argmin(1)
    near_tie = (np.sort(d, 1)[:, 1] - best) <= 2.0 ** -21 * np.maximum(best, 1e-30)
    cnt_exact = np.bincount(exact, minlength=7)
    assert int(cnt.sum()) == len(pts)
    assert np.abs(cnt.astype(np.int64) - cnt_exact).sum() <= 2 * int(near_tie.sum())
    if not near_tie.any():
        for j in range(7):
            sel = pts[exact == j].astype(np.float64)
            if len(sel):
                np.testing.assert_allclose(c_new[j], (sel.sum(0) / len(sel)).astype(np.float32), rtol=0, atol=0)


def test_km_k1_is_global_mean():
    rng = np.random.default_rng(7)
    pts, cen = _quantised(rng, 5000, 1)
    c_new, cnt = decode("km", oracle.run("km", [(pts.view(np.uint8).reshape(-1), None, len(pts), 32, 0)], centroids=cen))
    assert cnt.tolist() == [5000]
    exact = pts.astype(np.float64).mean(0)                 # quantised data: the fp64 sum is exact
    np.testing.assert_array_equal(c_new[0], exact.astype(np.float32))


def test_km_empty_cluster_keeps_centroid():
    pts = np.zeros((10, 8), np.float32)
    cen = np.array([[0] * 8, [100] * 8], np.float32)
    c_new, cnt = decode("km", oracle.run("km", [(pts.view(np.uint8).reshape(-1), None, 10, 32, 0)], centroids=cen))
    assert cnt.tolist() == [10, 0]
    np.testing.assert_array_equal(c_new[1], cen[1])


def test_km_tie_goes_to_lowest_id():
    pts = np.zeros((1, 8), np.float32)
    cen = np.array([[1] * 8, [-1] * 8, [1] * 8], np.float32)
    c_new, cnt = decode("km", oracle.run("km", [(pts.view(np.uint8).reshape(-1), None, 1, 32, 0)], centroids=cen))
    assert cnt.tolist() == [1, 0, 0]


def test_km_generator_blobs_exact_counts():
    spec = pygen.KMSpec()
    n = 32 * 2000
    pts = pygen.host_km(spec, n)
    c_blob, init = pygen.km_centres(spec)
    c_new, cnt = decode("km", oracle.run("km", [(pts.view(np.uint8).reshape(-1), None, n, 32, 0)], centroids=init))
    assert cnt.tolist() == [n // 32] * 32                      # blob of point i = i mod 32
    # invariant: Σ cnt_j c'_j ≈ Σ x   and exact fp64 means on quantised data
    for j in range(32):
        sel = pts[j::32].astype(np.float64)
        np.testing.assert_array_equal(c_new[j], (sel.sum(0) / len(sel)).astype(np.float32))
    assert np.all(np.abs(pts) < 128) and np.all(pts * 1024 == np.round(pts * 1024))


# ---------------- InvertedIndex ----------------
def brute_ii(recs, bases):
    out = {}
    for r, b in zip(recs, bases):
        start = 0
        while True:
            p = r.find(b'<a href="', start)
            if p < 0:
                break
            q = r.find(b'"', p + 9)
            if q > p + 9:
                out.setdefault(r[p + 9:q], []).append(b + p + 9)
            start = p + 1
    return {k: tuple(sorted(v)) for k, v in out.items()}


def test_ii_bruteforce_tiny():
    recs = [b'x<a href="u1">y<a href="u2">', b'<a href="">', b'<a href="u1', b'"', b'<a href="u1"<a href="u3"',
            b'<A HREF="u9">', b'<a name="u8">', b'', b'<a href="u2"']
    data, off = make_records(recs)
    got = decode("ii", oracle.run("ii", [(data, off, len(recs), 0, 50)]))
    exp = brute_ii(recs, [50 + int(o) for o in off[:-1]])
    assert got == exp
    assert set(got) == {b"u1", b"u2", b"u3"}


def test_ii_generator_ground_truth():
    spec = pygen.spec_ii(4)
    g = pygen.host_text(spec, 8, truth=True)
    got = decode("ii", oracle.run("ii", [(g["data"], g["offsets"], g["n"], 0, 0)]))
    exp = {}
    for v in g["links"].tolist():
        uid, off = v >> 40, v & ((1 << 40) - 1)
        exp.setdefault(pygen.url(uid), []).append(off)
    exp = {k: tuple(sorted(v)) for k, v in exp.items()}
    assert len(exp) > 500
    assert got == exp                                           # distractors produce nothing
    # Table II: ~7.94 records per URL occurrence
    occ = sum(len(v) for v in got.values())
    assert 6.5 < g["n"] / occ < 9.5


# ---------------- generator shape (weak pin, Table II) ----------------
def test_generator_table2_shapes():
    g = pygen.host_text(pygen.spec_wc(10_000, 1), 2)
    ll = np.diff(g["offsets"].astype(np.int64))
    assert abs(ll.mean() - 32.44) / 32.44 < 0.10 and abs(ll.std() - 2.59) / 2.59 < 0.10
    g = pygen.host_text(pygen.spec_sm(), 2)
    ll = np.diff(g["offsets"].astype(np.int64))
    assert abs(ll.mean() - 44.52) / 44.52 < 0.10 and abs(ll.std() - 2.68) / 2.68 < 0.10
    g = pygen.host_text(pygen.spec_ii(), 8)
    ll = np.diff(g["offsets"].astype(np.int64))
    assert abs(ll.mean() - 63.9) / 63.9 < 0.10 and abs(ll.std() - 123.2) / 123.2 < 0.15
