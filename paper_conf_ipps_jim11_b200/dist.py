"""Process-group plumbing for the multi-GPU exchange: byte-count exchange and
variable-size all-to-all over torch.distributed (NCCL on B200, gloo in the CPU tests).  No
MapReduce arithmetic here: libbmr's kernels produce and consume the buffers."""
from __future__ import annotations

import numpy as np


def exchange_counts(counts: np.ndarray, group=None) -> np.ndarray:
    """counts[r] = (entries, heap bytes) this rank sends to rank r -> recv[r] = what rank r sends
    to this rank.  One all_to_all_single of nranks x 2 int64."""
    import torch
    import torch.distributed as dist
    world = dist.get_world_size(group)
    assert counts.shape == (world, 2)
    dev = _dev(group)
    send = torch.from_numpy(np.ascontiguousarray(counts, np.int64)).to(dev)
    recv = torch.empty_like(send)
    dist.all_to_all_single(recv, send, group=group)
    return recv.cpu().numpy()


def alltoallv(send, send_bytes, recv_bytes, group=None):
    """Variable all-to-all of a flat uint8 tensor: slice r (send_bytes[r] bytes, in rank order)
    goes to rank r; returns the concatenation of what every rank sent here, in rank order."""
    import torch
    import torch.distributed as dist
    send_bytes = [int(x) for x in send_bytes]
    recv_bytes = [int(x) for x in recv_bytes]
    out = torch.empty(sum(recv_bytes), dtype=torch.uint8, device=send.device)
    if sum(send_bytes) == 0 and sum(recv_bytes) == 0:
        return out
    if send.is_cuda and dist.get_backend(group) != "nccl":   # gloo: staged through host memory
        tmp = torch.empty(sum(recv_bytes), dtype=torch.uint8)
        dist.all_to_all_single(tmp, send.cpu(), output_split_sizes=recv_bytes, input_split_sizes=send_bytes,
                               group=group)
        return tmp.to(send.device)
    dist.all_to_all_single(out, send, output_split_sizes=recv_bytes, input_split_sizes=send_bytes, group=group)
    return out


def _dev(group):
    import torch
    import torch.distributed as dist
    if dist.get_backend(group) == "nccl":
        return torch.device("cuda", torch.cuda.current_device())
    return torch.device("cpu")


def open_xwindows(own, group=None):
    """f-3 plumbing: every rank publishes the CUDA IPC handle of its own receive window (an
    XWindow(ipc=True)) with one all_gather_object; returns the rank-ordered window list for
    Job.set_xwindows (own window for this rank, mapped peer windows for the others).  Close the
    peer windows (XWindow.close) after the last Map that uses them."""
    import torch.distributed as dist
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    mine = (own.ipc_handle(), own.entry_cap, own.heap_cap)
    alls = [None] * world
    dist.all_gather_object(alls, mine, group=group)
    from . import XWindow
    return [own if r == rank else XWindow.open_peer(h, ec, hc, own.device) for r, (h, ec, hc) in enumerate(alls)]
