"""Multi-GPU plumbing: one process per GPU, torch.distributed for the
collectives, libsj.so for everything else.

The join partitions naturally: every unordered pair is evaluated by
exactly one query point, so queue slices produce disjoint pair sets and no pair ever
crosses a GPU.  The only exchanges are
  * one broadcast of the index blob (sj_export_index -> sj_create_from_index) from the
    rank that built it, over NCCL / NVLink on GPUs (gloo on CPU for the tests), and
  * one all-reduce of the per-rank counters.
Each rank then runs sj_set_slice(rank, world): queue chunk c (SJ_OPT_GRAB positions of
D', workload-sorted) belongs to rank c mod world, so every slice is itself
non-increasing in workload and the work per rank is balanced to within one chunk.
"""
from __future__ import annotations

import torch
import torch.distributed as dist

from ._lib import Handle


def broadcast_blob(blob: torch.Tensor | None, src: int = 0, group=None, device: str | torch.device = "cpu"):
    """Broadcast a uint8 blob from `src`; returns the blob on every rank (same device)."""
    rank = dist.get_rank(group)
    size = torch.zeros(1, dtype=torch.int64, device=device)
    if rank == src:
        size[0] = blob.numel()
    dist.broadcast(size, src, group=group)
    if rank != src:
        blob = torch.empty(int(size.item()), dtype=torch.uint8, device=device)
    dist.broadcast(blob, src, group=group)
    return blob


def allreduce_counts(values, group=None, device: str | torch.device = "cpu", op=dist.ReduceOp.SUM):
    """All-reduce a list of integer counters (int64)."""
    t = torch.tensor([int(v) for v in values], dtype=torch.int64, device=device)
    dist.all_reduce(t, op=op, group=group)
    return [int(x) for x in t.tolist()]


def replicate_index(handle: Handle | None, src: int = 0, group=None, device="cuda"):
    """Rank `src` exports its handle's index into a device blob, NCCL-broadcasts it, and every
    other rank builds a handle from it.  Returns (handle, blob)."""
    rank = dist.get_rank(group)
    blob = None
    if rank == src:
        nbytes = handle.export_index()
        blob = torch.empty(nbytes, dtype=torch.uint8, device=device)
        handle.export_index(blob, nbytes)
    blob = broadcast_blob(blob, src, group, device)
    if rank != src:
        handle = Handle.from_index(blob, blob.numel())
    return handle, blob


def distributed_self_join(points, eps: float, out, cap: int, group=None, src: int = 0, **options):
    """The multi-GPU hot path: build on `src`, replicate, join this rank's slice into `out`
    (device buffer of `cap` pairs), all-reduce {pairs, distance calcs}.
    Returns (handle, local_pairs, total_pairs)."""
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    dev = torch.device("cuda", torch.cuda.current_device())
    h = Handle(points, eps, **options) if rank == src else None
    h, _ = replicate_index(h, src, group, dev)
    if rank != src:
        for k, v in options.items():
            h.set_option(k, v)
    h.set_slice(rank, world)
    rc, local = h.self_join(out, cap)
    total = allreduce_counts([local], group, dev)[0]
    return h, local, total
