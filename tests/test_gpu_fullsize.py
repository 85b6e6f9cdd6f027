"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times (device-
resident input generated in HBM, one persistent CTA per SM), against properties that hold at
any size and are computed without the CUDA path:
  C5 WordCount 8 GiB  == generator ground truth (histogram of drawn word ranks, exact)
  C2 StringMatch 4 GiB == generator planted-offset set (exact)
  C3 KMeans 64M points: counts == n/32 per blob (exact) and centroids == fp64 blob means (1e-5)
  C4 InvertedIndex 8 GiB: sampled URLs == generator planted (URL, offset) lists (exact), and
     total occurrences == planted links
The oracle itself is run on sampled pages (C5) for an independent element-wise check."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import paper_conf_ipps_jim11_b200 as bmr  # noqa: E402
from gen import pygen  # noqa: E402
from oracle import oracle  # noqa: E402
from tests.helpers import decode  # noqa: E402


def run_dev(workload, g, **kw):
    with bmr.Job(workload, **kw) as job:
        job.map(g["data"], g["offsets"], g["n"])
        job.group()
        job.reduce()
        r = job.fetch()
        st = job.stats()
    return r, st


def test_c5_wordcount_8gib_vs_ground_truth():
    spec = pygen.spec_wc(1_000_000, 5)
    pages = 8192
    g = pygen.device_text(spec, pages)
    r, st = run_dev("wc", g)
    del g
    torch.cuda.empty_cache()
    hist = np.zeros(spec.vocab, np.uint64)
    for p0 in range(0, pages, 1024):                   # host truth in slices (bounded memory)
        h = pygen.host_text(spec, 1024, page0=p0, truth=True)
        hist += h["word_hist"].astype(np.uint64)
    ko, vo = r["key_offsets"], r["val_offsets"]
    keys, vals = bytes(r["keys"]), r["vals"].view(np.uint64)
    assert r["n_keys"] == int((hist > 0).sum())
    assert int(vals.sum()) == int(hist.sum()) == st["pairs"] + st["words_combined"]
    # every (word, count) equals the drawn-rank histogram (spellings are unique per rank)
    want = {pygen.word(i): int(c) for i in np.nonzero(hist)[0].tolist() for c in [hist[i]]}
    got = {keys[ko[i]:ko[i + 1]]: int(vals[i]) for i in range(r["n_keys"])}
    assert got == want


def test_c5_sampled_pages_vs_oracle():
    """element-wise check of the same code path on 64 sampled pages of the C5 shard"""
    spec = pygen.spec_wc(1_000_000, 5)
    rng = np.random.default_rng(0)
    for p0 in sorted(rng.choice(8192 - 8, 8, replace=False).tolist()):
        h = pygen.host_text(spec, 8, page0=p0)
        d = pygen.device_text(spec, 8, page0=p0)
        r, _ = run_dev("wc", d)
        assert decode("wc", r) == decode("wc", oracle.run("wc", [(h["data"], h["offsets"], h["n"], 0, 0)]))


def test_c2_stringmatch_4gib_vs_planted():
    spec = pygen.spec_sm(1000, 2)
    pages = 4096
    g = pygen.device_text(spec, pages)
    r, st = run_dev("sm", g, pattern=spec.pattern)
    del g
    plants = []
    for p0 in range(0, pages, 1024):
        plants.append(pygen.host_text(spec, 1024, page0=p0, truth=True)["plants"])
    plants = np.sort(np.concatenate(plants))
    got = decode("sm", r)
    assert len(got) > 50_000
    assert np.array_equal(got, plants)


def test_c3_kmeans_64m_blob_means():
    spec = pygen.KMSpec()
    n = 64 << 20
    pts = pygen.device_km(spec, n)
    _, init = pygen.km_centres(spec)
    with bmr.Job("km", centroids=init) as job:
        job.map(pts.view(-1).view(torch.uint8), None, n)
        job.group()
        job.reduce()
        cen, cnt = decode("km", job.fetch())
    assert cnt.tolist() == [n // 32] * 32                      # blob of point i = i mod 32
    # exact fp64 blob means (quantised coordinates: fp64 sums are exact)
    x = pts.view(n // 32, 32, 8).double().sum(0).cpu().numpy() / (n // 32)
    mean_abs = pts.abs().double().mean(0).cpu().numpy()
    assert np.all(np.abs(cen.astype(np.float64) - x) <= 1e-5 * np.maximum(np.abs(x), mean_abs[None]))


def test_c4_invindex_8gib_vs_planted_links():
    # ALL planted links of the 8 GiB input against generator truth: the same 16.7 M offsets, the
    # same grouping (one GPU key per URL id and vice versa), and the key bytes of a random sample
    # of 50k URLs (plus every URL with id % 97 == 0) spelled as the generator spells them
    spec = pygen.spec_ii(4)
    pages = 8192
    g = pygen.device_text(spec, pages)
    r, st = run_dev("ii", g)
    del g
    ko, vo = r["key_offsets"], r["val_offsets"]
    keys, vals = bytes(r["keys"]), r["vals"].view(np.uint64)
    nk = int(r["n_keys"])
    occ = int(vo[-1] // 8)
    links = np.concatenate([pygen.host_text(spec, 1024, page0=p0, truth=True)["links"]
                            for p0 in range(0, pages, 1024)])
    assert occ == len(links) == st["pairs"]
    t_off = links & np.uint64((1 << 40) - 1)
    t_id = links >> np.uint64(40)
    o_t = np.argsort(t_off, kind="stable")
    t_off, t_id = t_off[o_t], t_id[o_t]
    g_key = np.repeat(np.arange(nk, dtype=np.int64), np.diff(vo // 8).astype(np.int64))
    o_g = np.argsort(vals, kind="stable")
    g_off, g_key = vals[o_g], g_key[o_g]
    assert np.array_equal(g_off, t_off)                       # every link found, none invented
    pairs = np.unique(np.stack([g_key, t_id.astype(np.int64)], 1), axis=0)
    assert len(pairs) == nk == len(np.unique(t_id))          # grouping == URL ids, a bijection
    key_of_id = dict(zip(pairs[:, 1].tolist(), pairs[:, 0].tolist()))
    rng = np.random.default_rng(4)
    ids = set(rng.choice(pairs[:, 1], 50_000, replace=False).tolist())
    ids |= {int(u) for u in pairs[:, 1] if u % 97 == 0}
    for u in ids:
        i = key_of_id[u]
        assert keys[ko[i]:ko[i + 1]] == pygen.url(u)
