"""Host-side logic of the multi-GPU exchange on CPU: world_size-2 gloo process
group, 127.0.0.1 rendezvous.  Checks the count exchange and the variable all-to-all that move
libbmr's partition buffers between ranks (the device kernels are covered by
tests/test_gpu_multirank.py with a loopback exchange on one GPU)."""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch.distributed as dist
    from paper_conf_ipps_jim11_b200 import dist as D
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        rng = np.random.default_rng(rank)
        # rank r sends to rank d: (entries = 3 + r + 2d, heap = 8 * (r + d)) with recognisable bytes
        counts = np.array([[3 + rank + 2 * d, 8 * (rank + d)] for d in range(world)], np.int64)
        eb = 16
        ent = torch.cat([torch.full((int(counts[d, 0]) * eb,), 10 * rank + d, dtype=torch.uint8) for d in range(world)])
        heap = torch.cat([torch.full((int(counts[d, 1]),), 100 + 10 * rank + d, dtype=torch.uint8) for d in range(world)])
        recv = D.exchange_counts(counts)
        exp = np.array([[3 + s + 2 * rank, 8 * (s + rank)] for s in range(world)], np.int64)
        assert np.array_equal(recv, exp), (recv, exp)
        r_ent = D.alltoallv(ent, counts[:, 0] * eb, recv[:, 0] * eb)
        r_heap = D.alltoallv(heap, counts[:, 1], recv[:, 1])
        off = 0
        for s in range(world):                       # concatenated in source-rank order
            n = int(recv[s, 0]) * eb
            assert torch.all(r_ent[off:off + n] == 10 * s + rank)
            off += n
        off = 0
        for s in range(world):
            n = int(recv[s, 1])
            assert torch.all(r_heap[off:off + n] == 100 + 10 * s + rank)
            off += n
        # empty exchange is a no-op
        z = np.zeros((world, 2), np.int64)
        assert D.alltoallv(torch.zeros(0, dtype=torch.uint8), z[:, 0], D.exchange_counts(z)[:, 0]).numel() == 0
        q.put((rank, "ok"))
    except Exception as e:  # pragma: no cover
        q.put((rank, repr(e)))
        raise
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_exchange_plumbing_gloo(world):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(120)
    res = dict(q.get(timeout=5) for _ in range(world))
    assert all(v == "ok" for v in res.values()), res
    assert all(p.exitcode == 0 for p in procs)
