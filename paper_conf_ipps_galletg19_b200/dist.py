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


def replicate_index(handle: Handle | None, src: int = 0, group=None, device="cuda", view: bool | None = None):
    """Rank `src` exports its handle's index into a device blob, NCCL-broadcasts it, and every
    other rank builds a handle from it -- by default (device blobs) a zero-copy VIEW whose index
    arrays are the broadcast buffer itself (sj_create_from_index_view: no allocation, no copy;
    the handle keeps the blob alive).  Returns (handle, blob)."""
    rank = dist.get_rank(group)
    blob = None
    if rank == src:
        nbytes = handle.export_index()
        blob = torch.empty(nbytes, dtype=torch.uint8, device=device)
        handle.export_index(blob, nbytes)
    blob = broadcast_blob(blob, src, group, device)
    if rank != src:
        if view is None:
            view = blob.is_cuda
        handle = Handle.from_index(blob, blob.numel(), view=view)
    return handle, blob


def replicated_self_join(points, eps: float, out, cap: int, group=None, **options):
    """The multi-GPU path for inputs every rank holds (the bench's replicated input): every rank
    builds the same index from its own copy (the build is deterministic: identical D', chunks and
    slices on every rank), joins its WorkQueue slice (chunk c -> rank c mod world) into `out`,
    and one all-reduce sums the pairs.  No broadcast: the build runs on all ranks at once instead
    of on one rank followed by a 100+ MB broadcast.  Returns (handle, local_pairs, total)."""
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    h = Handle(points, eps, **options)
    h.set_slice(rank, world)
    rc, local = h.self_join(out, cap)
    dev = out.device if hasattr(out, "device") else torch.device("cpu")
    total = allreduce_counts([local], group, dev)[0]
    return h, local, total


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
# sets of the ranks are disjoint and their union is the global join.
#
# Every piece of the cut's arithmetic -- bounds, the dimension-0 cell column of every point,
# the column histogram, slab ownership, the halo selection and the packing of the rows per
# destination -- runs in libsj (sj_part_*, csrc/partition.cu).  This module only moves data
# between the calls with collectives: an all-reduce of the bounds, an all-reduce of the column
# histogram and two all-to-alls (own rows, halo rows) -- NCCL over NVLink on GPUs.  The router
# argument lets the CPU tests drive the same collective plumbing with gloo and a reference
# router (tests/slab_ref.py); the product path always uses LibRouter.


class LibRouter:
    """The slab arithmetic of libsj (sj_part_*): device tensors in, device tensors out."""

    def bounds(self, points):
        from ._lib import sj_part_bounds
        return sj_part_bounds(points)

    def columns(self, origin0: float, max0: float, eps: float) -> int:
        from ._lib import sj_part_columns
        return sj_part_columns(origin0, max0, eps)

    def histogram(self, points, origin0: float, eps: float, ncol: int):
        from ._lib import sj_part_histogram
        return sj_part_histogram(points, origin0, eps, ncol)

    def pack(self, points, ids, origin0: float, eps: float, hist, world: int):
        from ._lib import sj_part_pack
        return sj_part_pack(points, ids, origin0, eps, hist, world)


def _host_staged(group) -> bool:
    """gloo (the CPU tests, several processes sharing one GPU) moves CUDA tensors through host
    memory; NCCL takes them as they are."""
    return dist.get_backend(group) == "gloo"


def _all_reduce(t: torch.Tensor, op, group=None) -> torch.Tensor:
    if t.is_cuda and _host_staged(group):
        c = t.cpu()
        dist.all_reduce(c, op=op, group=group)
        return c.to(t.device)
    dist.all_reduce(t, op=op, group=group)
    return t


def _exchange(rows: torch.Tensor, ids: torch.Tensor, counts, group=None):
    """all_to_all of packed rows (grouped by destination rank, `counts` rows each) and their
    ids; returns the rows and ids this rank receives, ordered by source rank."""
    world = len(counts)
    if rows.is_cuda and _host_staged(group):
        r, i = _exchange(rows.cpu(), ids.cpu(), counts, group)
        return r.to(rows.device), i.to(rows.device)
    dev = rows.device
    dim = rows.shape[1]
    scount = torch.tensor([int(c) for c in counts], dtype=torch.int64, device=dev)
    rcount = torch.empty_like(scount)
    dist.all_to_all_single(rcount, scount, group=group)
    sc, rc = scount.tolist(), rcount.tolist()
    out = torch.empty((sum(rc), dim), dtype=rows.dtype, device=dev)
    out_ids = torch.empty(sum(rc), dtype=ids.dtype, device=dev)
    dist.all_to_all_single(out, rows[: sum(sc)].contiguous(), rc, sc, group=group)
    dist.all_to_all_single(out_ids, ids[: sum(sc)].contiguous(), rc, sc, group=group)
    assert world == dist.get_world_size(group)
    return out, out_ids


def slab_partition(points: torch.Tensor, ids: torch.Tensor, eps: float, group=None, router=None):
    """This rank's partition of a self-join whose points are spread over the ranks.
    points: (n_local, dim) float64, ids: (n_local,) int32 global ids (the uint32 bits) on the
    device the collectives run on.  Returns (part_points, part_ids int32, n_query, origin list):
    own points first, then the halo."""
    router = router or LibRouter()
    world = dist.get_world_size(group)
    dim = points.shape[1]
    mn, mx = router.bounds(points)
    mn = torch.tensor(mn, dtype=torch.float64, device=points.device)
    mx = torch.tensor(mx, dtype=torch.float64, device=points.device)
    mn = _all_reduce(mn, dist.ReduceOp.MIN, group)
    mx = _all_reduce(mx, dist.ReduceOp.MAX, group)
    origin = [float(v) for v in mn.tolist()]
    ncol = router.columns(origin[0], float(mx[0].item()), eps)
    hist = _all_reduce(router.histogram(points, origin[0], eps, ncol), dist.ReduceOp.SUM, group)
    own_p, own_i, own_c, halo_p, halo_i, halo_c = router.pack(points, ids, origin[0], eps, hist, world)
    mine, mine_ids = _exchange(own_p, own_i, own_c, group)
    halo, halo_ids = _exchange(halo_p, halo_i, halo_c, group)
    part = torch.cat([mine, halo], 0) if halo.shape[0] else mine
    part_ids = torch.cat([mine_ids, halo_ids], 0) if halo.shape[0] else mine_ids
    assert part.shape[1] == dim
    return part, part_ids, int(mine.shape[0]), origin


def partitioned_self_join(points: torch.Tensor, ids: torch.Tensor, eps: float, group=None, **options):
    """Spatially partitioned multi-GPU join: slab_partition, then this rank's partitioned handle
    joins into a device buffer sized by its count.  points / ids (int32 global ids) on this
    rank's GPU.  Returns (pairs (m, 2) int32 holding uint32 global ids, local pair count,
    all-reduced total)."""
    from ._lib import self_join_pairs

    dev = points.device
    ppts, pids, nq, origin = slab_partition(points, ids, eps, group)
    if ppts.shape[0] == 0:  # an empty slab (more ranks than occupied cell columns)
        pairs = torch.empty((0, 2), dtype=torch.int32, device=dev)
    else:
        with Handle(ppts, eps, part=(pids, nq, origin), **options) as h:
            pairs = self_join_pairs(h, dev)
    local = int(pairs.shape[0])
    total = allreduce_counts([local], group, dev)[0]
    return pairs, local, total
