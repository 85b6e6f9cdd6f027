"""Can two processes on ONE GPU form an NCCL communicator (each rank pretending to be its own
host: NCCL_HOSTID differs, so NCCL's duplicate-GPU check passes and the ranks talk through the
socket transport over loopback)?"""
import os, sys
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def run(rank, world, port):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), NCCL_HOSTID=f"bmrhost{rank}",
                      NCCL_SOCKET_IFNAME="lo", NCCL_IB_DISABLE="1", NCCL_DEBUG=os.environ.get("NCCL_DEBUG", "WARN"))
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", rank=rank, world_size=world, device_id=torch.device("cuda:0"))
    t = torch.full((4,), float(rank + 1), device="cuda")
    dist.all_reduce(t)
    x = torch.arange(8, device="cuda", dtype=torch.int64) + 100 * rank
    y = torch.empty_like(x)
    dist.all_to_all_single(y, x)
    torch.cuda.synchronize()
    print(f"rank {rank}: allreduce {t.tolist()} a2a {y.tolist()}", flush=True)
    dist.destroy_process_group()


if __name__ == "__main__":
    mp.spawn(run, args=(2, 29533), nprocs=2)
