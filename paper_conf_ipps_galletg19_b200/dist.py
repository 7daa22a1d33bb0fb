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


# ----------------------------------------------------------------------------- spatial slabs
# SURVEY §8(f)4 (beyond replication; not in the paper): instead of replicating the whole
# index, the ranks own SLABS of whole cell columns along dimension 0.  LID-UNICOMP (P:174,
# Alg. 3) only looks at cells whose dimension-0 coordinate is the same or one higher, so a
# slab needs, besides its own points, only the points of the first cell column of the next
# non-empty slab (the halo).  Each rank builds a partitioned handle (sj_create_part: queries =
# own points, halo = candidates, the global grid origin, global ids) and joins it; the pair
# sets of the ranks are disjoint and their union is the global join.  Exchanges: an all-reduce
# of the per-dimension bounds, an all-reduce of the column histogram, and two all-to-alls
# (own points, halo points) -- NCCL over NVLink on GPUs, gloo in the CPU tests.

def cell_width(eps: float) -> float:
    """Cell side w = eps(1 + 2^-20) (reading c5), in binary64 like the library."""
    return float(eps) * (1.0 + 2.0 ** -20)


def cell_columns(x0: torch.Tensor, origin0: float, eps: float) -> torch.Tensor:
    """Dimension-0 cell coordinate floor(fl(fl(x - origin) / w)) (IEEE binary64 RN, one
    subtraction and one division: the library's a3 arithmetic), as int64."""
    return torch.floor((x0 - origin0) / cell_width(eps)).to(torch.int64)


def slab_owners(hist: torch.Tensor, world: int) -> torch.Tensor:
    """Owner rank of every cell column: columns are dealt to ranks in order, a column wholly to
    the rank in whose share (by point count) its first point falls -- slabs of whole columns,
    balanced to within one column.  hist: points per column (int64)."""
    total = int(hist.sum().item())
    if total == 0:
        return torch.zeros_like(hist)
    start = torch.cumsum(hist, 0) - hist  # global position of each column's first point
    return torch.clamp((start * world) // total, max=world - 1)


def _all_to_all(x: torch.Tensor, dest: torch.Tensor, world: int, group=None):
    """Send row i of x to rank dest[i]; returns the rows this rank receives (ordered by source
    rank, stable within a source)."""
    order = torch.argsort(dest, stable=True)
    send = x[order].contiguous()
    scount = torch.bincount(dest, minlength=world).to(torch.int64)
    rcount = torch.empty_like(scount)
    dist.all_to_all_single(rcount, scount, group=group)
    sc, rc = scount.tolist(), rcount.tolist()
    out = torch.empty((sum(rc),) + tuple(x.shape[1:]), dtype=x.dtype, device=x.device)
    dist.all_to_all_single(out, send, rc, sc, group=group)
    return out


def slab_partition(points: torch.Tensor, ids: torch.Tensor, eps: float, group=None):
    """This rank's partition of a self-join whose points are spread over the ranks.
    points: (n_local, dim) float64, ids: (n_local,) int64 global ids (any device; collectives run
    there).  Returns (part_points, part_ids int64, n_query, origin list): own points first,
    then the halo."""
    world = dist.get_world_size(group)
    dev = points.device
    dim = points.shape[1]
    inf = torch.full((dim,), float("inf"), dtype=torch.float64, device=dev)
    mn = points.min(0).values if points.shape[0] else inf
    mx = points.max(0).values if points.shape[0] else -inf
    dist.all_reduce(mn, op=dist.ReduceOp.MIN, group=group)
    dist.all_reduce(mx, op=dist.ReduceOp.MAX, group=group)
    origin = [float(v) for v in mn.tolist()]
    ncol = int(cell_columns(mx[:1], origin[0], eps).item()) + 1
    col = cell_columns(points[:, 0], origin[0], eps)
    hist = torch.bincount(col, minlength=ncol).to(torch.int64)
    dist.all_reduce(hist, group=group)
    owner = slab_owners(hist, world)
    own = owner[col]
    # halo: a column's points also go to the owner of the column before it, if that differs
    prev = owner[torch.clamp(col - 1, min=0)]
    hsel = (col >= 1) & (prev != own)
    rows = torch.cat([points, ids.to(torch.float64).unsqueeze(1)], 1)  # ids < 2^32: exact in binary64
    mine = _all_to_all(rows, own, world, group)
    halo = _all_to_all(rows[hsel], prev[hsel], world, group)
    part = torch.cat([mine, halo], 0)
    return part[:, :dim].contiguous(), part[:, dim].to(torch.int64), int(mine.shape[0]), origin


def partitioned_self_join(points: torch.Tensor, ids: torch.Tensor, eps: float, group=None, **options):
    """Spatially partitioned multi-GPU join: slab_partition, then this rank's partitioned handle
    joins into a device buffer sized by its count.  Returns (pairs (m, 2) int32 holding uint32
    global ids, local pair count, all-reduced total)."""
    from ._lib import self_join_pairs

    dev = torch.device("cuda", torch.cuda.current_device())
    ppts, pids, nq, origin = slab_partition(points, ids, eps, group)
    ids32 = (pids & 0xFFFFFFFF).to(torch.int32)  # the library reads the bits as uint32
    if ppts.shape[0] == 0:  # an empty slab (more ranks than occupied cell columns)
        pairs = torch.empty((0, 2), dtype=torch.int32, device=dev)
    else:
        with Handle(ppts.to(dev), eps, part=(ids32.to(dev), nq, origin), **options) as h:
            pairs = self_join_pairs(h, dev)
    local = int(pairs.shape[0])
    total = allreduce_counts([local], group, points.device)[0]
    return pairs, local, total
