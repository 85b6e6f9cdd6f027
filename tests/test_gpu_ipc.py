"""Fused Map flush + shuffle across PROCESSES: two ranks on one GPU, each
with its own process, publish their receive windows through CUDA IPC handles (gloo
all_gather_object, as dist.open_xwindows does over NCCL on a multi-GPU box), every rank's Map
stores its InvertedIndex records straight into the owner's window, then each rank ingests its own
window, groups and reduces.  The union of the two outputs must equal the oracle."""
import os
import pickle
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

PAGES = 6


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, out_dir):
    import torch
    import torch.distributed as dist
    import paper_conf_ipps_jim11_b200 as bmr
    from paper_conf_ipps_jim11_b200 import dist as D
    from gen import pygen
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    spec = pygen.spec_ii(4)
    a, b = rank * PAGES // world, (rank + 1) * PAGES // world
    g = pygen.host_text(spec, b - a, page0=a)
    own = bmr.XWindow(1 << 20, 64 << 20, ipc=True)
    wins = D.open_xwindows(own)
    job = bmr.Job("ii", rank=rank, nranks=world, input_base=g["base"])
    job.set_xwindows(wins)
    d = torch.from_numpy(g["data"]).cuda()
    o = torch.from_numpy(g["offsets"].view(np.int64)).cuda()
    job.map(d, o, g["n"])
    torch.cuda.synchronize()
    dist.barrier()                      # every rank's records are in their windows
    job.ingest_xwindow(own)
    job.group()
    job.reduce()
    res = job.fetch()
    with open(os.path.join(out_dir, f"r{rank}.pkl"), "wb") as f:
        pickle.dump({k: (np.asarray(v) if not np.isscalar(v) else v) for k, v in res.items()}, f)
    job.close()
    dist.barrier()                      # no rank stores into a peer window any more
    for w in wins:
        if w is not own:
            w.close()
    dist.barrier()
    own.close()
    dist.destroy_process_group()


def test_ii_fused_ipc_two_processes(tmp_path):
    import torch.multiprocessing as mp
    from gen import pygen
    from oracle import oracle
    from tests.helpers import decode
    world = 2
    mp.start_processes(_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, start_method="spawn",
                       join=True)
    got = {}
    for r in range(world):
        with open(tmp_path / f"r{r}.pkl", "rb") as f:
            d = decode("ii", pickle.load(f))
        assert not (set(d) & set(got)), "a key reached two ranks"
        got.update(d)
    whole = pygen.host_text(pygen.spec_ii(4), PAGES)
    exp = decode("ii", oracle.run("ii", [(whole["data"], whole["offsets"], whole["n"], 0, 0)]))
    assert got == exp
