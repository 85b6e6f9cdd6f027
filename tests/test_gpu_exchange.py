"""The multi-GPU exchange (SURVEY §8(b) mr_group with R > 1, §8(e)) across PROCESSES on one GPU:
R ranks, each with its byte-range shard, run map -> group (-> exchange) -> reduce; the union of
the rank outputs must equal the oracle over the whole input, for both exchanges —
  * "nccl": libbmr's own (mr_comm_init + cfg.nccl_comm: ncclAlltoAll of the counts, one NCCL
    group of send/recv), each rank its own NCCL host so NCCL accepts them on one GPU;
  * "shuffle": the caller-moved one (Job.shuffle: mr_partition_count / _write, torch.distributed
    all-to-all over gloo staged through host memory, mr_ingest).
Each rank runs the job twice on the same mr_job (reset in between: buffer reuse after an
ingest), and both runs must give the same result."""
import os
import pickle
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import paper_conf_ipps_jim11_b200 as bmr  # noqa: E402
from gen import pygen  # noqa: E402
from oracle import oracle  # noqa: E402
from tests.helpers import decode  # noqa: E402
from tests import mp_exchange  # noqa: E402


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def run_ranks(mode, workload, R, flags, units, tmp_path, timeout=240, nbatch=1):
    ctx = torch.multiprocessing.get_context("spawn")
    port = _free_port()
    ps = [ctx.Process(target=mp_exchange.worker, args=(r, R, port, mode, workload, flags, units, str(tmp_path), nbatch))
          for r in range(R)]
    for p in ps:
        p.start()
    for p in ps:
        p.join(timeout)
    for p in ps:
        if p.is_alive():
            p.kill()
    assert all(p.exitcode == 0 for p in ps), [p.exitcode for p in ps]
    return [pickle.load(open(os.path.join(tmp_path, f"r{r}.pkl"), "rb")) for r in range(R)]


def union(outs, workload):
    u = {}
    for r in outs:
        d = decode(workload, r)
        assert not (set(d) & set(u)), "a key reached two ranks"
        u.update(d)
    return u


def whole(workload, units):
    if workload == "km":
        pts = pygen.host_km(pygen.KMSpec(), units)
        return pts, oracle.run("km", [(pts.view(np.uint8).reshape(-1), None, units, 32, 0)],
                               centroids=pygen.km_centres(pygen.KMSpec())[1])
    spec = pygen.spec_wc(1_000_000, 5) if workload == "wc" else pygen.spec_ii(4)
    g = pygen.host_text(spec, units)
    return g, oracle.run(workload, [(g["data"], g["offsets"], g["n"], 0, 0)])


CASES = [("wc", 0, 4), ("wc", bmr.FLAG_NO_COMBINE, 4), ("ii", 0, 6)]


@pytest.mark.parametrize("mode", ["nccl", "shuffle"])
@pytest.mark.parametrize("workload,flags,units", CASES, ids=["wc-combine", "wc-raw", "ii"])
def test_exchange_text(mode, workload, flags, units, tmp_path):
    R = 3 if mode == "nccl" else 2
    res = run_ranks(mode, workload, R, flags, units, tmp_path)
    _, ref = whole(workload, units)
    exp = decode(workload, ref)
    for step in range(2):
        got = union([r["outs"][step] for r in res], workload)
        assert got == exp, f"step {step}"
    if mode == "nccl":
        assert sum(r["stats"][1]["xchg_send_bytes"] for r in res) == sum(r["stats"][1]["xchg_recv_bytes"] for r in res) > 0


def test_exchange_batch_combine(tmp_path):
    # strong-scaling shape: every rank folds its shard batch by batch
    # (MR_FLAG_BATCH_COMBINE), then the merged partials go through the NCCL exchange
    res = run_ranks("nccl", "wc", 2, bmr.FLAG_BATCH_COMBINE, 6, tmp_path, nbatch=3)
    exp = decode("wc", whole("wc", 6)[1])
    for step in range(2):
        assert union([r["outs"][step] for r in res], "wc") == exp


@pytest.mark.parametrize("mode", ["nccl", "shuffle"])
def test_exchange_km(mode, tmp_path):
    R, units = 2, 32 * 3000
    res = run_ranks(mode, "km", R, 0, units, tmp_path)
    pts, ref = whole("km", units)
    co, no = decode("km", ref)
    floor = np.abs(pts.astype(np.float64)).mean(0)
    for step in range(2):
        cen = np.zeros((32, 8), np.float32)
        cnt = np.zeros(32, np.uint64)
        seen = set()
        for r in res:
            o = r["outs"][step]
            ko, vo = o["key_offsets"], o["val_offsets"]
            for i in range(o["n_keys"]):
                j = int(np.frombuffer(bytes(o["keys"][ko[i]:ko[i + 1]]), np.uint32)[0])
                assert j not in seen
                seen.add(j)
                v = bytes(o["vals"][vo[i]:vo[i + 1]])
                cen[j] = np.frombuffer(v[:32], np.float32)
                cnt[j] = np.frombuffer(v[32:40], np.uint64)[0]
        assert seen == set(range(32))
        assert np.array_equal(cnt, no)
        assert np.all(np.abs(cen.astype(np.float64) - co) <= 1e-5 * np.maximum(np.abs(co), floor[None]))
