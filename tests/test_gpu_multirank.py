"""Multi-GPU group-by on ONE GPU: R virtual ranks, each with its own job and
byte-range shard, partition their records, a loopback exchange routes the slices (the same
bytes NCCL would move), every rank ingests, groups and reduces its own keys; the union of the
rank outputs must equal the oracle over the whole input (R-rank == 1-rank == oracle)."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import paper_conf_ipps_jim11_b200 as bmr  # noqa: E402
from gen import pygen  # noqa: E402
from oracle import oracle  # noqa: E402
from tests.helpers import decode  # noqa: E402


def shards_text(spec, npages, R):
    """page-aligned byte-range shards: rank r gets pages [r*P/R, (r+1)*P/R)"""
    out = []
    for r in range(R):
        a, b = r * npages // R, (r + 1) * npages // R
        out.append(pygen.host_text(spec, b - a, page0=a))
    return out


def run_virtual(workload, shards, R, **kw):
    jobs, keep, parts = [], [], []
    for r in range(R):
        g = shards[r]
        extra = dict(kw)
        if workload in ("sm", "ii"):
            extra["input_base"] = g["base"]
        job = bmr.Job(workload, rank=r, nranks=R, **extra)
        if workload == "km":
            d = torch.from_numpy(g["data"]).cuda()
            keep.append(d)
            job.map(d, None, g["n"])
        else:
            d = torch.from_numpy(g["data"]).cuda()
            o = torch.from_numpy(g["offsets"].view(np.int64)).cuda()
            keep.append((d, o))
            job.map(d, o, g["n"])
        parts.append(job.partition())
        jobs.append(job)
    outs = []
    for dst in range(R):
        ents, heaps, rc = [], [], np.zeros((R, 2), np.int64)
        for src in range(R):
            ent, heap, counts, eb = parts[src]
            e0 = int(counts[:dst, 0].sum()) * eb
            h0 = int(counts[:dst, 1].sum())
            ents.append(ent[e0:e0 + int(counts[dst, 0]) * eb])
            heaps.append(heap[h0:h0 + int(counts[dst, 1])])
            rc[src] = counts[dst]
        ent_d = torch.cat(ents) if ents else torch.zeros(0, dtype=torch.uint8, device="cuda")
        heap_d = torch.cat(heaps) if heaps else torch.zeros(0, dtype=torch.uint8, device="cuda")
        jobs[dst].ingest(ent_d, heap_d, rc)
        keep.append((ent_d, heap_d))
    for job in jobs:
        job.group()
        job.reduce()
        outs.append(job.fetch())
        job.close()
    return outs


def union_dict(outs, workload):
    u = {}
    for r in outs:
        d = decode(workload, r)
        assert not (set(d) & set(u)), "a key reached two ranks"
        u.update(d)
    return u


@pytest.mark.parametrize("R", [1, 2, 3, 4])
@pytest.mark.parametrize("flags", [0, bmr.FLAG_NO_COMBINE], ids=["combine", "raw"])
def test_wc_multirank(R, flags):
    spec = pygen.spec_wc(1_000_000, 5)
    sh = shards_text(spec, 4, R)
    got = union_dict(run_virtual("wc", sh, R, flags=flags), "wc")
    whole = pygen.host_text(spec, 4)
    exp = decode("wc", oracle.run("wc", [(whole["data"], whole["offsets"], whole["n"], 0, 0)]))
    assert got == exp


@pytest.mark.parametrize("R", [2, 4])
def test_ii_multirank(R):
    spec = pygen.spec_ii(4)
    sh = shards_text(spec, 6, R)
    got = union_dict(run_virtual("ii", sh, R), "ii")
    whole = pygen.host_text(spec, 6)
    exp = decode("ii", oracle.run("ii", [(whole["data"], whole["offsets"], whole["n"], 0, 0)]))
    assert got == exp


@pytest.mark.parametrize("R", [2, 3])
def test_km_multirank(R):
    spec = pygen.KMSpec()
    n = 32 * 3000
    pts = pygen.host_km(spec, n)
    _, init = pygen.km_centres(spec)
    shards = []
    for r in range(R):
        a, b = r * n // R, (r + 1) * n // R
        shards.append({"data": pts[a:b].view(np.uint8).reshape(-1).copy(), "n": b - a})
    outs = run_virtual("km", shards, R, centroids=init)
    cen = np.zeros((32, 8), np.float32)
    cnt = np.zeros(32, np.uint64)
    seen = set()
    for r in outs:
        ko, vo = r["key_offsets"], r["val_offsets"]
        for i in range(r["n_keys"]):
            j = int(np.frombuffer(bytes(r["keys"][ko[i]:ko[i + 1]]), np.uint32)[0])
            assert j not in seen
            seen.add(j)
            v = bytes(r["vals"][vo[i]:vo[i + 1]])
            cen[j] = np.frombuffer(v[:32], np.float32)
            cnt[j] = np.frombuffer(v[32:40], np.uint64)[0]
    assert seen == set(range(32))
    co, no = decode("km", oracle.run("km", [(pts.view(np.uint8).reshape(-1), None, n, 32, 0)], centroids=init))
    assert np.array_equal(cnt, no)
    floor = np.abs(pts.astype(np.float64)).mean(0)
    assert np.all(np.abs(cen.astype(np.float64) - co) <= 1e-5 * np.maximum(np.abs(co), floor[None]))


def run_fused_ii(shards, R, entry_cap=1 << 20, heap_cap=64 << 20):
    """f-3: every rank's Map appends its records straight into the destination ranks' receive
    windows (here all on one GPU); after all Maps, every rank ingests its own window."""
    wins = [bmr.XWindow(entry_cap, heap_cap) for _ in range(R)]
    jobs, keep = [], []
    for r in range(R):
        g = shards[r]
        job = bmr.Job("ii", rank=r, nranks=R, input_base=g["base"])
        job.set_xwindows(wins)
        d = torch.from_numpy(g["data"]).cuda()
        o = torch.from_numpy(g["offsets"].view(np.int64)).cuda()
        keep.append((d, o))
        job.map(d, o, g["n"])
        jobs.append(job)
    torch.cuda.synchronize()   # every rank's Map (and so every window) is complete
    return jobs, wins, keep


@pytest.mark.parametrize("R", [1, 2, 3])
def test_ii_fused_xwindows(R):
    spec = pygen.spec_ii(4)
    sh = shards_text(spec, 6, R)
    jobs, wins, keep = run_fused_ii(sh, R)
    outs = []
    for r in range(R):
        jobs[r].ingest_xwindow(wins[r])
    for job in jobs:
        job.group()
        job.reduce()
        outs.append(job.fetch())
        job.close()
    got = union_dict(outs, "ii")
    whole = pygen.host_text(spec, 6)
    res = oracle.run("ii", [(whole["data"], whole["offsets"], whole["n"], 0, 0)])
    exp = decode("ii", res)
    assert got == exp
    # every record left through a window, and only there
    assert sum(w.used()[0] for w in wins) == sum(len(v) for v in exp.values())
    # the same records as the partition + all-to-all path
    assert got == union_dict(run_virtual("ii", sh, R), "ii")


def test_ii_fused_xwindow_overflow():
    spec = pygen.spec_ii(4)
    sh = shards_text(spec, 2, 2)
    jobs, wins, keep = run_fused_ii(sh, 2, entry_cap=16, heap_cap=1 << 20)
    with pytest.raises(bmr.MRError, match="MR_ERR_OOM"):
        jobs[0].ingest_xwindow(wins[0])
    for job in jobs:
        job.close()
