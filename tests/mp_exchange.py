"""Worker of tests/test_gpu_exchange.py (importable by spawned processes): one rank of a
multi-process job on cuda:0.  Each rank is its own NCCL "host" (NCCL_HOSTID), so NCCL accepts
several ranks on one GPU and connects them through its socket transport over loopback; the
exchange itself is libbmr's (mr_group with nccl_comm) or the caller-moved one (Job.shuffle over
a gloo group, staged through host memory).  Every rank runs the job TWICE on the same mr_job
(reset between) and returns both fetched results."""
import os
import pickle
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def shard(workload, r, R, units):
    from gen import pygen
    import numpy as np
    if workload == "km":
        a, b = r * units // R, (r + 1) * units // R
        pts = pygen.host_km(pygen.KMSpec(), units)[a:b]
        return {"data": pts.view(np.uint8).reshape(-1).copy(), "offsets": None, "n": b - a, "base": 0}
    spec = pygen.spec_wc(1_000_000, 5) if workload == "wc" else pygen.spec_ii(4)
    a, b = r * units // R, (r + 1) * units // R
    return pygen.host_text(spec, b - a, page0=a)


def worker(rank, world, port, mode, workload, flags, units, outdir, nbatch=1):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), NCCL_HOSTID=f"bmrtest{rank}",
                      NCCL_SOCKET_IFNAME="lo", NCCL_IB_DISABLE="1")
    if ROOT not in sys.path:
        sys.path.insert(0, ROOT)
    import numpy as np
    import torch
    import torch.distributed as dist
    import paper_conf_ipps_jim11_b200 as bmr
    from gen import pygen
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        g = shard(workload, rank, world, units)
        comm = bmr.Comm.from_torch() if mode == "nccl" else None
        kw = dict(rank=rank, nranks=world, comm=comm, flags=flags)
        if workload == "km":
            kw["centroids"] = pygen.km_centres(pygen.KMSpec())[1]
        if workload == "ii":
            kw["input_base"] = g["base"]
        # nbatch > 1 (text): the shard is mapped as consecutive record batches
        cuts = [g["n"] * i // nbatch for i in range(nbatch + 1)]
        batches = []
        for a, c in zip(cuts, cuts[1:]):
            if g["offsets"] is None:
                batches.append((torch.from_numpy(g["data"][a * 32:c * 32]).cuda(), None, c - a))
            else:
                off = g["offsets"]
                batches.append((torch.from_numpy(g["data"][int(off[a]):int(off[c])]).cuda(),
                                torch.from_numpy((off[a:c + 1] - off[a]).view(np.int64)).cuda(), c - a))
        outs, stats = [], []
        with bmr.Job(workload, **kw) as job:
            for _ in range(2):
                job.reset()
                for d, o, n in batches:
                    job.map(d, o, n)
                if mode == "shuffle":
                    job.shuffle()
                job.group()
                job.reduce()
                outs.append(job.fetch())
                stats.append(job.stats())
        with open(os.path.join(outdir, f"r{rank}.pkl"), "wb") as f:
            pickle.dump({"outs": outs, "stats": stats}, f)
        if comm is not None:
            comm.close()
    finally:
        dist.destroy_process_group()
