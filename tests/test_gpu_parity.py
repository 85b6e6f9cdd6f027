"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, element by element
after the C-1 canonicalisation, on seeded inputs that span several tiles with ragged tails,
plus the edge cases of each workload.  Integer workloads are bit-exact; KMeans counts are
exact and centroids within the DESIGN.md §5 tolerance (1e-5 relative, floor = mean |x|)."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import paper_conf_ipps_jim11_b200 as bmr  # noqa: E402
from gen import pygen  # noqa: E402
from oracle import oracle  # noqa: E402
from tests.helpers import decode, make_records  # noqa: E402

KM_RTOL = 1e-5


def dev(data, off=None):
    d = torch.from_numpy(np.ascontiguousarray(data)).cuda()
    o = None if off is None else torch.from_numpy(np.ascontiguousarray(off).view(np.int64)).cuda()
    return d, o


def gpu(workload, batches, **kw):
    """batches: [(data u8, offsets u64 or None, n)] host arrays -> decoded GPU result + stats."""
    keep = []
    with bmr.Job(workload, **kw) as job:
        for data, off, n in batches:
            d, o = dev(data, off)
            keep.append((d, o))
            job.map(d, o, n)
        job.group()
        job.reduce()
        r = job.fetch()
        st = job.stats()
    return r, st


def ora(workload, batches, **kw):
    ob, base = [], 0
    for data, off, n in batches:
        ob.append((data, off, n, 32 if off is None else 0, base))
        base += len(data)
    return oracle.run(workload, ob, **kw)


def same(workload, batches, gkw=None, okw=None):
    g, st = gpu(workload, batches, **(gkw or {}))
    o = ora(workload, batches, **(okw or {}))
    dg, do = decode(workload, g), decode(workload, o)
    if workload == "sm":
        assert np.array_equal(dg, do)
    else:
        assert dg == do
    # WC: words absorbed by the in-SMEM combiner are not emitted as pairs
    assert st["pairs"] + st["words_combined"] == o["pairs"]
    return dg, st


# ------------------------------------------------------------------ WordCount
def test_wc_c1_parity_and_ground_truth():
    g = pygen.host_text(pygen.spec_wc(10_000, 1), 1, truth=True)
    got, st = same("wc", [(g["data"], g["offsets"], g["n"])])
    exp = {pygen.word(i): int(c) for i, c in enumerate(g["word_hist"]) if c}
    assert got == exp


def test_wc_multi_tile_v1m():
    g = pygen.host_text(pygen.spec_wc(1_000_000, 5), 3)
    same("wc", [(g["data"], g["offsets"], g["n"])])


def _wc_edge_records(seed):
    rng = np.random.default_rng(seed)
    recs = []
    alpha = list(b"abcXYZ019 ,.;\n\x80\xff")
    total = 0
    while total < 70_000:                                  # > 4 tiles of 16 KiB
        kind = rng.integers(0, 10)
        if kind == 0:
            r = b""
        elif kind == 1:
            r = bytes(rng.choice(list(b"abcdefgh"), size=int(rng.integers(20, 400))).tolist())  # long word
        elif kind == 2:
            r = b"x" * 7 + b" " + b"y" * 8 + b" " + b"z" * 9    # inline / hashed boundary
        else:
            r = bytes(rng.choice(alpha, size=int(rng.integers(0, 60))).tolist())
        recs.append(r)
        total += len(r)
    recs.append(b"q" * 20_000)                              # word spanning > one tile + halo
    recs.append(b"tail" * 3)
    return recs


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_wc_edge_cases_ragged(seed):
    data, off = make_records(_wc_edge_records(seed))
    same("wc", [(data, off, len(off) - 1)])


@pytest.mark.parametrize("shift", [1, 3, 8, 13])
def test_wc_unaligned_records(shift):
    data, off = make_records(_wc_edge_records(7))
    d = torch.zeros(len(data) + 32, dtype=torch.uint8, device="cuda")
    d[shift:shift + len(data)] = torch.from_numpy(data).cuda()
    o = torch.from_numpy(off.view(np.int64)).cuda()
    with bmr.Job("wc") as job:
        job.map(d[shift:shift + len(data)], o, len(off) - 1)
        job.group(); job.reduce()
        r = job.fetch()
    assert decode("wc", r) == decode("wc", ora("wc", [(data, off, len(off) - 1)]))


def test_wc_empty_inputs():
    for recs in ([], [b""], [b"", b"", b""], [b" ,.\n"]):
        data, off = make_records(recs)
        got, st = same("wc", [(data, off, len(recs))])
        assert got == {}


def test_wc_single_words_and_record_boundaries():
    recs = [b"ab", b"cd", b"", b"e f", b"gh", b"longerword12345", b"A" * 33]
    data, off = make_records(recs)
    same("wc", [(data, off, len(recs))])


def test_wc_force_tiny_out_and_weak_hash(monkeypatch):
    g = pygen.host_text(pygen.spec_wc(1_000_000, 5), 2)
    b = [(g["data"], g["offsets"], g["n"])]
    base, _ = same("wc", b)
    tiny, st = same("wc", b, gkw={"flags": bmr.FLAG_FORCE_TINY_OUT | bmr.FLAG_NO_MAP_COMBINE})
    assert st["flushes"] > 500            # 641-unit buffers instead of 3068
    tiny2, _ = same("wc", b, gkw={"flags": bmr.FLAG_FORCE_TINY_OUT})
    assert tiny2 == tiny
    # the hashed stream (words > 8 symbols without the L2 tables, which count words of <= 16
    # symbols exactly): a 4-bit hash forces collisions, the byte verification must split them
    monkeypatch.setenv("BMR_TABLE_MIN_BYTES", str(1 << 40))
    weak, st2 = same("wc", b, gkw={"flags": bmr.FLAG_WEAK_HASH_DEBUG})
    assert st2["collisions"] > 0          # verification found the forced collisions
    assert base == tiny == weak


def test_wc_map_combiner_on_and_off():
    # f-1: the in-SMEM combiner absorbs most repeated short words; the result must not depend on it
    g = pygen.host_text(pygen.spec_wc(1_000_000, 5), 24)
    b = [(g["data"], g["offsets"], g["n"])]
    on, st_on = same("wc", b)
    off, st_off = same("wc", b, gkw={"flags": bmr.FLAG_NO_MAP_COMBINE})
    assert on == off
    assert st_off["words_combined"] == 0 and st_off["pairs_partial"] == 0
    # (with the L2 tables every exact and mid word is counted there: words_combined, no partial pairs)
    assert st_on["words_combined"] > st_on["pairs"] // 4
    assert st_on["pairs"] + st_on["words_combined"] == st_off["pairs"]


def test_wc_small_input_sort_path(monkeypatch):
    # below BMR_TABLE_MIN_BYTES the exact words take the sorted exact stream + SMEM-combiner
    # partials (no L2 tables): same result, and the partials are pairs this time
    g = pygen.host_text(pygen.spec_wc(1_000_000, 5), 24)
    b = [(g["data"], g["offsets"], g["n"])]
    monkeypatch.setenv("BMR_TABLE_MIN_BYTES", str(1 << 40))
    small, st = same("wc", b)
    monkeypatch.setenv("BMR_TABLE_MIN_BYTES", "0")
    big, st2 = same("wc", b)
    assert small == big and st["pairs_partial"] > 0 and st2["pairs_partial"] == 0


def test_wc_combiner_partials_replay_and_multibatch(monkeypatch):
    # tiny capacities: the exact, partial and hashed streams all overflow and the batches replay
    # (the streams: no L2 tables)
    monkeypatch.setenv("BMR_TABLE_MIN_BYTES", str(1 << 40))
    g = pygen.host_text(pygen.spec_wc(10_000, 3), 3)
    data, off = g["data"], g["offsets"]
    cuts = [0, g["n"] // 4, g["n"] // 2, g["n"]]
    b = [(data[int(off[a]):int(off[c])], off[a:c + 1] - off[a], c - a) for a, c in zip(cuts, cuts[1:])]
    got, st = same("wc", b, gkw={"max_pairs_hint": 2000})
    assert st["replays"] >= 3 and st["words_combined"] > 0
    assert got == decode("wc", ora("wc", [(data, off, g["n"])]))


MODES = {"SO": bmr.FLAG_NO_SMEM_IN, "SI": bmr.FLAG_NO_SMEM_OUT, "G": bmr.FLAG_NO_SMEM_IN | bmr.FLAG_NO_SMEM_OUT}


@pytest.mark.parametrize("mode", sorted(MODES))
def test_memory_modes_wc_ii_sm(mode):
    # f-2: the paper's memory-usage modes (SO / SI / G, L129-135, L171-175) on the same kernel
    # give the SIO result for every text workload, incl. ragged tails and capacity replays
    f = MODES[mode]
    g = pygen.host_text(pygen.spec_wc(1_000_000, 5), 3)
    b = [(g["data"], g["offsets"], g["n"])]
    assert same("wc", b, gkw={"flags": f})[0] == same("wc", b)[0]
    same("wc", b, gkw={"flags": f, "max_pairs_hint": 5000})
    data, off = make_records(_mixed_length_records(9, 3000))
    same("wc", [(data, off, len(off) - 1)], gkw={"flags": f | bmr.FLAG_NO_MAP_COMBINE})
    gi = pygen.host_text(pygen.spec_ii(4), 2)
    same("ii", [(gi["data"], gi["offsets"], gi["n"])], gkw={"flags": f})
    spec = pygen.spec_sm(plant_ppm=50_000)
    gs = pygen.host_text(spec, 2, truth=True)
    got, _ = same("sm", [(gs["data"], gs["offsets"], gs["n"])], gkw={"pattern": spec.pattern, "flags": f},
                  okw={"pattern": spec.pattern})
    assert np.array_equal(got, gs["plants"])


@pytest.mark.parametrize("mode", sorted(MODES))
def test_memory_modes_km(mode):
    spec = pygen.KMSpec()
    pts = pygen.host_km(spec, 32 * 700 + 3)
    _, init = pygen.km_centres(spec)
    km_check(pts, init, flags=MODES[mode])
    km_check(pts, init, flags=MODES[mode] | bmr.FLAG_NO_MAP_COMBINE)


@pytest.mark.parametrize("chunk", [None, 100_000, 4_096])
def test_map_host_lines_equals_offsets(chunk, monkeypatch):
    # mr_map_host_lines: the device-derived line directory (in batches overlapped with the copies)
    # gives the same result as the host offsets, incl. an unterminated last line and lines longer
    # than a batch
    if chunk:
        monkeypatch.setenv("BMR_LINE_CHUNK", str(chunk))
    g = pygen.host_text(pygen.spec_wc(1_000_000, 5), 2)
    text = np.concatenate([g["data"], np.frombuffer(b"tail words " * 700 + b"no newline", np.uint8)])
    off = np.concatenate([g["offsets"], np.array([len(text)], np.uint64)])
    n = len(off) - 1
    for wl, kw in (("wc", {}), ("ii", {}), ("sm", {"pattern": b"tail words tail "})):
        with bmr.Job(wl, **kw) as job:
            job.map_host_lines(text)
            job.group()
            job.reduce()
            got = decode(wl, job.fetch())
            st = job.stats()
        want = decode(wl, ora(wl, [(text, off, n)], **({"pattern": kw["pattern"]} if wl == "sm" else {})))
        if wl == "sm":
            assert np.array_equal(got, want) and len(got) > 0
        else:
            assert got == want
        assert st["input_bytes"] == len(text)


def test_wc_replay_on_overflow(monkeypatch):
    monkeypatch.setenv("BMR_TABLE_MIN_BYTES", str(1 << 40))   # (pair streams, no L2 tables)
    g = pygen.host_text(pygen.spec_wc(10_000, 1), 1)
    got, st = same("wc", [(g["data"], g["offsets"], g["n"])], gkw={"max_pairs_hint": 1000})
    assert st["replays"] >= 1


def _mixed_length_records(seed, n):
    """Words of 1..14 symbols over [0-9A-Za-z] (exact keys <= 7 bytes, hashed beyond), with
    repeats, so both WordCount streams and the 6-bit alnum packing are exercised."""
    rng = np.random.default_rng(seed)
    alpha = np.frombuffer(b"0123456789ABCDEFGHIJKLMNOPQRSTUVWXYZabcdefghijklmnopqrstuvwxyz", np.uint8)
    vocab = [bytes(alpha[rng.integers(0, 62, size=L)]) for L in rng.integers(1, 15, size=400)]
    vocab += [b"0" * L for L in range(1, 15)] + [b"z" * L for L in range(1, 15)] + [b"Z9a0Yb", b"Z9a0Yb1"]
    recs = []
    for _ in range(n):
        k = int(rng.integers(0, 12))
        recs.append(b" ".join(vocab[int(i)] for i in rng.integers(0, len(vocab), size=k)))
    return recs


def test_wc_exact_and_hashed_streams():
    data, off = make_records(_mixed_length_records(5, 3000))
    got, st = same("wc", [(data, off, len(off) - 1)])
    lens = {len(k) for k in got}
    assert min(lens) == 1 and max(lens) >= 12 and {6, 7} <= lens


def test_wc_hashed_stream_replay(monkeypatch):
    # every word is longer than 8 bytes: without the L2 tables the whole Map output is the hashed
    # stream
    monkeypatch.setenv("BMR_TABLE_MIN_BYTES", str(1 << 40))
    recs = [b" ".join(b"w%08d" % (i * 7 + j) for j in range(5)) for i in range(4000)]
    data, off = make_records(recs)
    got, st = same("wc", [(data, off, len(recs))], gkw={"max_pairs_hint": 1000})
    assert st["replays"] >= 1 and len(got) == 20000


@pytest.mark.parametrize("fmt", [b"L%011d", b"x%016d"], ids=["12-symbol", "17-symbol"])
def test_wc_long_words_table_and_stream(fmt):
    # 300k distinct words of 12 symbols (long-word table: more than its first 2^18 slots hold ->
    # grow + replay) or of 17 symbols (> 16: the hashed stream), twice each
    words = [fmt % i for i in range(300_000)]
    recs = [b" ".join(words[i:i + 6]) for i in range(0, len(words), 6)] * 2
    data, off = make_records(recs)
    got, st = same("wc", [(data, off, len(recs))])
    assert len(got) == 300_000 and set(got.values()) == {2}
    if len(words[0]) <= 16:
        assert st["replays"] >= 1 and st["pairs_hashed"] == 0
    else:
        assert st["pairs_hashed"] == 600_000


def test_wc_mid_table_growth_replay():
    # 400k distinct 7-symbol words (mid keys) twice each: more than the first mid table holds
    # within its probe bound -> the Map flags it, the table grows 4x and the batch is replayed
    words = [b"m%06d" % i for i in range(400_000)]
    recs = [b" ".join(words[i:i + 8]) for i in range(0, len(words), 8)] * 2
    data, off = make_records(recs)
    got, st = same("wc", [(data, off, len(recs))])
    assert st["replays"] >= 1 and len(got) == 400_000 and set(got.values()) == {2}


def test_wc_multibatch():
    g = pygen.host_text(pygen.spec_wc(1000, 11), 2)
    data, off = g["data"], g["offsets"]
    cut = g["n"] // 3
    b0 = (data[: int(off[cut])], off[: cut + 1], cut)
    b1 = (data[int(off[cut]):], off[cut:] - off[cut], g["n"] - cut)
    got, _ = same("wc", [b0, b1])
    assert got == decode("wc", ora("wc", [(data, off, g["n"])]))


@pytest.mark.parametrize("flags", [0, bmr.FLAG_NO_MAP_COMBINE], ids=["map-combiner", "no-map-combiner"])
def test_wc_batch_combine(flags):
    # MR_FLAG_BATCH_COMBINE ("batched processing at another level"): every batch is
    # grouped + reduced when the next one is mapped; mr_group merges the (key, count) partials
    g = pygen.host_text(pygen.spec_wc(1_000_000, 5), 10)
    data, off = g["data"], g["offsets"]
    cuts = [0, g["n"] // 5, g["n"] // 2, g["n"] // 2 + 1, g["n"]]
    b = [(data[int(off[a]):int(off[c])], off[a:c + 1] - off[a], c - a) for a, c in zip(cuts, cuts[1:])]
    exp = decode("wc", ora("wc", [(data, off, g["n"])]))
    for f in (bmr.FLAG_BATCH_COMBINE | flags, flags):
        r, st = gpu("wc", b, flags=f)
        assert decode("wc", r) == exp
        assert st["n_keys"] == len(exp)
    # the job is reusable after a folded run (reset keeps the buffers, clears the partials)
    keep = []
    with bmr.Job("wc", flags=bmr.FLAG_BATCH_COMBINE | flags) as job:
        for _ in range(2):
            job.reset()
            for data_b, off_b, n in b:
                d, o = dev(data_b, off_b)
                keep.append((d, o))
                job.map(d, o, n)
            job.group()
            job.reduce()
            assert decode("wc", job.fetch()) == exp


@pytest.mark.parametrize("workload", ["ii", "km", "sm"])
def test_overflow_spill_under_forced_congestion(workload):
    # MR_FLAG_FORCE_TINY_OUT: every warp result fills an output buffer; with MR_FLAG_FORCE_SPILL
    # every overflowing warp result is written straight to HBM (map_spills, §8(a) a5) instead of
    # waiting for the next buffer (the default spills only while the ring is congested) — the
    # output must not change
    if workload == "ii":
        g = pygen.host_text(pygen.spec_ii(4), 6)
        b, kw = [(g["data"], g["offsets"], g["n"])], {}
    elif workload == "sm":
        spec = pygen.spec_sm(260_000, 2)                 # dense plants: > 512 matches per CTA
        g = pygen.host_text(spec, 24)
        b, kw = [(g["data"], g["offsets"], g["n"])], {"pattern": spec.pattern}
    else:
        spec = pygen.KMSpec()
        n = 32 * 20_000
        pts = pygen.host_km(spec, n)
        b, kw = [(pts.view(np.uint8).reshape(-1), None, n)], {"centroids": pygen.km_centres(spec)[1]}
    okw = dict(kw)
    flags = bmr.FLAG_FORCE_TINY_OUT | bmr.FLAG_FORCE_SPILL | (bmr.FLAG_NO_MAP_COMBINE if workload == "km" else 0)
    if workload == "km":
        r, st = gpu("km", b, flags=flags, **kw)
        cen, cnt = decode("km", r)
        co, no = decode("km", ora("km", b, **okw))
        assert np.array_equal(cnt, no)
    else:
        _, st = same(workload, b, gkw=dict(flags=flags, **kw), okw=okw)
    assert st["map_spills"] > 0, st


# ------------------------------------------------------------------ StringMatch
def test_sm_generator_dense_plants():
    spec = pygen.spec_sm(plant_ppm=260_000)            # paper-shaped dense variant (3.83:1)
    g = pygen.host_text(spec, 3, truth=True)
    got, _ = same("sm", [(g["data"], g["offsets"], g["n"])], gkw={"pattern": spec.pattern},
                  okw={"pattern": spec.pattern})
    assert np.array_equal(got, g["plants"])


def test_sm_self_overlap_and_boundaries():
    pat = b"a" * 16
    recs = [b"a" * 1000, b"a" * 15, b"a" * 16, b"", b"b" + b"a" * 40, b"a" * 20_000]
    data, off = make_records(recs)
    got, _ = same("sm", [(data, off, len(recs))], gkw={"pattern": pat}, okw={"pattern": pat})
    assert len(got) == 985 + 0 + 1 + 25 + (20_000 - 15)


def test_sm_short_records_offsets_from_global():
    # ~4-byte records: > 512 record starts per 16 KiB tile, so the producers read the tile's
    # offsets from global memory instead of staging them (StringMatch stages at most 512)
    rng = np.random.default_rng(7)
    pat = b"#needle:0123456#"
    recs = [bytes(rng.integers(97, 100, size=int(rng.integers(0, 8)), dtype=np.uint8)) for _ in range(60_000)]
    for i in rng.choice(len(recs), 300, replace=False).tolist():
        recs[i] = b"x" + pat + b"y"
    data, off = make_records(recs)
    got, _ = same("sm", [(data, off, len(recs))], gkw={"pattern": pat}, okw={"pattern": pat})
    assert len(got) == 300


@pytest.mark.parametrize("flags", [0, bmr.FLAG_NO_SMEM_IN | bmr.FLAG_NO_SMEM_OUT], ids=["SIO", "G"])
def test_sm_per_line_output(flags):
    # f-4: the paper's own StringMatch output (L125: emit the line if found) = oracle "sml"
    pat = b"a" * 16
    recs = [b"a" * 1000, b"a" * 15, b"a" * 16, b"", b"b" + b"a" * 40, b"xyz" * 50, b"a" * 20_000, b"a" * 17]
    rng = np.random.default_rng(3)
    recs += [bytes(rng.choice(list(b"ab"), size=int(rng.integers(0, 40)), p=[0.9, 0.1]).tolist()) for _ in range(3000)]
    data, off = make_records(recs)
    half = len(recs) // 2
    b = [(data[: int(off[half])], off[: half + 1], half), (data[int(off[half]):], off[half:] - off[half], len(recs) - half)]
    g, st = gpu("sm", b, pattern=pat, flags=bmr.FLAG_SM_LINES | flags, input_base=5)
    o = oracle.run("sml", [(data, off, len(recs), 0, 5)], pattern=pat)
    got, want = decode("sm", g), decode("sm", o)
    assert np.array_equal(got, want) and len(want) > 5
    assert st["n_keys"] == len(want) and st["pairs"] >= len(want)


def test_sm_input_base_and_multibatch():
    spec = pygen.spec_sm(plant_ppm=50_000)
    g = pygen.host_text(spec, 2, truth=True)
    data, off = g["data"], g["offsets"]
    cut = g["n"] // 2
    b0 = (data[: int(off[cut])], off[: cut + 1], cut)
    b1 = (data[int(off[cut]):], off[cut:] - off[cut], g["n"] - cut)
    got, _ = same("sm", [b0, b1], gkw={"pattern": spec.pattern}, okw={"pattern": spec.pattern})
    assert np.array_equal(got, g["plants"])
    r, _ = gpu("sm", [(data, off, g["n"])], pattern=spec.pattern, input_base=1 << 40)
    assert np.array_equal(decode("sm", r), g["plants"] + np.uint64(1 << 40))


# ------------------------------------------------------------------ KMeans
def km_check(pts, cen, **gkw):
    data = pts.view(np.uint8).reshape(-1)
    r, st = gpu("km", [(data, None, len(pts))], centroids=cen, **gkw)
    o = ora("km", [(data, None, len(pts))], centroids=cen)
    cg, ng = decode("km", r)
    co, no = decode("km", o)
    assert np.array_equal(ng, no)                      # counts exact
    floor = np.abs(pts.astype(np.float64)).mean(0) if len(pts) else np.zeros(8)
    tol = KM_RTOL * np.maximum(np.abs(co.astype(np.float64)), floor[None, :])
    assert np.all(np.abs(cg.astype(np.float64) - co) <= tol)
    return cg, ng


def test_km_generator_blobs():
    spec = pygen.KMSpec()
    n = 32 * 4000 + 17                                  # ragged tail
    pts = pygen.host_km(spec, n)
    _, init = pygen.km_centres(spec)
    _, cnt = km_check(pts, init)
    assert int(cnt.sum()) == n


@pytest.mark.parametrize("flags", [0, bmr.FLAG_NO_MAP_COMBINE], ids=["combiner", "sorted"])
@pytest.mark.parametrize("k", [1, 7, 32, 64, 65, 300])
def test_km_random_quantised(k, flags):
    # k <= 64: the Map's in-SMEM combiner (f-1) unless NO_MAP_COMBINE; k > 64: sort + reduce
    rng = np.random.default_rng(k)
    pts = (rng.integers(-60_000, 60_000, size=(20_000, 8)) / 1024.0).astype(np.float32)
    cen = (rng.integers(-60_000, 60_000, size=(k, 8)) / 1024.0).astype(np.float32)
    km_check(pts, cen, flags=flags)


def test_km_combiner_multibatch():
    spec = pygen.KMSpec()
    pts = pygen.host_km(spec, 32 * 3000 + 5)
    _, init = pygen.km_centres(spec)
    data = pts.view(np.uint8).reshape(-1)
    cut = 32 * 1234 * 32
    b = [(data[:cut], None, cut // 32), (data[cut:], None, len(pts) - cut // 32)]
    r, st = gpu("km", b, centroids=init)
    assert st["pairs"] == 0 and st["words_combined"] == len(pts)
    o = ora("km", [(data, None, len(pts))], centroids=init)
    cg, ng = decode("km", r)
    co, no = decode("km", o)
    assert np.array_equal(ng, no)
    floor = np.abs(pts.astype(np.float64)).mean(0)
    assert np.all(np.abs(cg.astype(np.float64) - co) <= KM_RTOL * np.maximum(np.abs(co), floor[None, :]))


def km_pair(pts, cen, flags=0):
    data = pts.view(np.uint8).reshape(-1)
    r, _ = gpu("km", [(data, None, len(pts))], centroids=cen, flags=flags)
    return decode("km", r)


def _near_bisector_points(rng, cen, n):
    # points on / just off the bisector of random centroid pairs (the bound test must fail there
    # or decide exactly as the full scan): m + t (c_b - c_a) for t in a few ulps-to-1e-4 around 0
    a = rng.integers(0, len(cen), n)
    b = (a + 1 + rng.integers(0, len(cen) - 1, n)) % len(cen)
    m = (cen[a].astype(np.float64) + cen[b]) / 2
    t = rng.choice([0.0, 1e-7, -1e-7, 1e-6, -1e-6, 1e-5, -1e-5, 1e-4, -1e-4, 0.3, -0.3], n)
    return (m + t[:, None] * (cen[b].astype(np.float64) - cen[a])).astype(np.float32)


@pytest.mark.parametrize("case", ["blobs", "bisectors", "duplicates", "k1"])
def test_km_bound_test_equals_full_scan(case):
    # the default Map assigns a point to its lane's previous winner when the triangle-inequality
    # bound holds; MR_FLAG_KM_FULL_SCAN scans every centroid.  Same assignments ->
    # bit-identical output, and both equal the oracle (counts exact).
    rng = np.random.default_rng(7)
    spec = pygen.KMSpec()
    if case == "blobs":
        pts = pygen.host_km(spec, 32 * 2000 + 9)
        cen = pygen.km_centres(spec)[1]
    elif case == "bisectors":
        cen = (rng.integers(-4096, 4096, size=(32, 8)) / 64.0).astype(np.float32)
        pts = _near_bisector_points(rng, cen, 40_000)
        pts[::7] = cen[rng.integers(0, 32, len(pts[::7]))]   # exactly on a centroid
    elif case == "duplicates":
        cen = (rng.integers(-64, 64, size=(16, 8))).astype(np.float32)
        cen[5] = cen[3]
        cen[9] = cen[3]                                      # coincident centroids: ties -> lowest id
        pts = np.concatenate([cen[rng.integers(0, 16, 5000)] + rng.normal(0, 2, (5000, 8)),
                              _near_bisector_points(rng, cen, 5000)]).astype(np.float32)
    else:
        cen = np.array([[1.5] * 8], np.float32)
        pts = rng.normal(0, 10, (10_000, 8)).astype(np.float32)
    cb, nb = km_pair(pts, cen)
    cf, nf = km_pair(pts, cen, bmr.FLAG_KM_FULL_SCAN)
    assert np.array_equal(nb, nf)
    assert np.array_equal(cb.view(np.uint32), cf.view(np.uint32))
    km_check(pts, cen)


def test_km_empty_and_tiny():
    cen = np.array([[0] * 8, [100] * 8], np.float32)
    km_check(np.zeros((0, 8), np.float32), cen)
    km_check(np.ones((3, 8), np.float32), cen)


def test_km_force_tiny_out():
    spec = pygen.KMSpec()
    pts = pygen.host_km(spec, 32 * 500)
    _, init = pygen.km_centres(spec)
    km_check(pts, init, flags=bmr.FLAG_FORCE_TINY_OUT | bmr.FLAG_NO_MAP_COMBINE)


# ------------------------------------------------------------------ InvertedIndex
def test_ii_generator_parity_and_truth():
    spec = pygen.spec_ii(4)
    g = pygen.host_text(spec, 4, truth=True)
    got, _ = same("ii", [(g["data"], g["offsets"], g["n"])])
    exp = {}
    for v in g["links"].tolist():
        exp.setdefault(pygen.url(v >> 40), []).append(v & ((1 << 40) - 1))
    assert got == {k: tuple(sorted(v)) for k, v in exp.items()}


def test_ii_edge_cases():
    recs = [b'x<a href="u1">y<a href="u2">', b'<a href="">', b'<a href="u1', b'"', b'<a href="u1"<a href="u3"',
            b'<A HREF="u9">', b'<a name="u8">', b'', b'<a href="u2"', b'<a href="' + b"L" * 3000 + b'"',
            b"z" * 16370 + b'<a href="' + b"crossing-the-tile-boundary" * 30 + b'"',
            b'<a href="short">' * 50]
    data, off = make_records(recs)
    same("ii", [(data, off, len(recs))])
    same("ii", [(data, off, len(recs))], gkw={"flags": bmr.FLAG_WEAK_HASH_DEBUG | bmr.FLAG_FORCE_TINY_OUT})


# ------------------------------------------------------------------ radix sort
@pytest.mark.parametrize("n,bits", [(1, 64), (4095, 64), (4097, 8), (100_003, 64), (1 << 20, 20)])
def test_sort_u64_matches_stable_sort(n, bits):
    g = torch.Generator(device="cuda").manual_seed(n)
    k = torch.randint(-(1 << 62), 1 << 62, (n,), device="cuda", generator=g, dtype=torch.int64)
    if bits < 64:
        k = k & ((1 << bits) - 1)
    ks, perm = bmr.sort_u64(k)
    # unsigned order == signed order after flipping the sign bit; torch stable sort as reference
    flip = k ^ torch.tensor(-(1 << 63), dtype=torch.int64, device="cuda")
    ref_v, ref_i = torch.sort(flip, stable=True)
    assert torch.equal(perm.long(), ref_i)
    assert torch.equal(ks, k[ref_i])


def test_wc_job_reuse_across_sizes():
    """A job reused across runs of different sizes (grow-only buffers sized by the previous run:
    segment starts, sort workspaces, combiner partials) stays exact."""
    small = pygen.host_text(pygen.spec_wc(1_000_000, 5), 1)
    big = pygen.host_text(pygen.spec_wc(1_000_000, 5), 6)
    with bmr.Job("wc") as job:
        outs = []
        for g in (small, small, big, big):
            d, o = dev(g["data"], g["offsets"])
            job.reset()
            job.map(d, o, g["n"])
            job.group()
            job.reduce()
            outs.append(decode("wc", job.fetch()))
    assert outs[0] == outs[1] == decode("wc", ora("wc", [(small["data"], small["offsets"], small["n"])]))
    assert outs[2] == outs[3] == decode("wc", ora("wc", [(big["data"], big["offsets"], big["n"])]))
