"""Task partitioning of one query's stream across GPUs (one process per GPU).

SURVEY.md §8(e): consecutive query tasks are independent except for windows
that straddle a task boundary; the paper assembles those from fragments of
adjacent tasks in task-id order.  Across GPUs
the stream is cut into contiguous partitions; rank r emits exactly the windows
[closed(r-1), closed(r)) -- those closed by its own last tuple but not by its
predecessor's -- so the concatenation of the ranks' result streams in rank
order is the single-GPU result, with no gather.

The only exchange is the *halo*: rank r-1 sends rank r the raw tail tuples
that windows >= closed(r-1) need (fewer than s tuples for count windows; at
most one window span for time windows), plus the two integers
(closed(r-1), halo_first).  It runs once, before any compute, over
torch.distributed (NCCL on GPUs, gloo on CPU); this module only plans and moves
bytes -- every window is computed by libsaber's kernels on the owning GPU.
"""
from __future__ import annotations

from .saber import partition_plan


def partition_bounds(n_total: int, world: int, rank: int) -> tuple[int, int]:
    """Contiguous partition [begin, end) of n_total tuples for `rank`."""
    per = n_total // world
    b = rank * per
    e = n_total if rank == world - 1 else b + per
    return b, e


def exchange_halo(spec, part, begin: int, n: int, rank: int, world: int, plan=None):
    """Send this partition's halo to rank+1 and receive the predecessor's.

    ``part`` is a torch uint8 tensor holding this rank's n tuples (CUDA tensor
    with NCCL, CPU tensor with gloo).  Returns (halo, first_window, base_index):
    ``halo`` is a uint8 tensor of tuples to prepend (empty on rank 0),
    ``first_window`` the first window id this rank emits and ``base_index`` the
    global position of the first tuple it will submit (count windows).
    ``plan(spec, part, begin, n) -> (closed, halo_first)`` defaults to
    saber_partition_plan on the device (the window-closing rule lives in the
    library; CPU tests pass their own, computed from the oracle).
    """
    import torch
    import torch.distributed as dist

    tb = spec["schema"]["tuple_bytes"]
    dev = part.device
    ops = []
    if rank < world - 1:
        if plan is not None:
            closed, halo_first = plan(spec, part, begin, n)
        elif part.is_cuda:
            closed, halo_first = partition_plan(spec, part.data_ptr(), begin, n)
        else:
            raise ValueError("host partitions need an explicit plan (the library plans on the device)")
        meta_out = torch.tensor([closed, halo_first], dtype=torch.int64, device=dev)
        ops.append(dist.P2POp(dist.isend, meta_out, rank + 1))
    meta_in = torch.zeros(2, dtype=torch.int64, device=dev)
    if rank > 0:
        ops.append(dist.P2POp(dist.irecv, meta_in, rank - 1))
    if ops:
        for r in dist.batch_isend_irecv(ops):
            r.wait()
    ops = []
    if rank < world - 1:
        lo = (halo_first - begin) * tb
        if lo < 0:
            raise ValueError("halo reaches beyond the predecessor partition")
        tail = part[lo:n * tb]
        if tail.numel():
            ops.append(dist.P2POp(dist.isend, tail.contiguous(), rank + 1))
    halo = torch.empty(0, dtype=torch.uint8, device=dev)
    first_window, base_index = 0, begin
    if rank > 0:
        first_window, base_index = int(meta_in[0]), int(meta_in[1])
        hn = (begin - base_index) * tb
        halo = torch.empty(hn, dtype=torch.uint8, device=dev)
        if hn:
            ops.append(dist.P2POp(dist.irecv, halo, rank - 1))
    if ops:
        for r in dist.batch_isend_irecv(ops):
            r.wait()
    return halo, first_window, base_index
