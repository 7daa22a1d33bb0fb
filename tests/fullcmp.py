"""Element-by-element comparison of a GPU pair list with the oracle at full size (test helper).

The GPU result (an (P, 2) int32 CUDA tensor of uint32 ids, in whatever order the join wrote it)
is cut into slabs of 2^27 pairs; each slab's canonical keys i << 32 | j are sorted on the device
and split by query-id block.  Each block's pieces are merged and sorted again, copied to the host
and compared with the oracle's rows of the same queries (oracle.Grid.keys_range: O2, the full
3^n scan, each row ascending), i.e. the whole pair list in canonical (i, j) order, block by block,
so neither side ever holds more than one block on the host.
"""
from __future__ import annotations

import numpy as np

import oracle

SLAB = 1 << 27


def canonical_blocks_equal(pairs_dev, pts, eps, block_pairs: int = 100_000_000, grid=None):
    """Asserts that the GPU pair list equals the oracle's, element by element after canonical
    sorting.  Returns (total pairs, number of blocks)."""
    import torch

    n = pts.shape[0]
    total = int(pairs_dev.shape[0])
    nb = max(1, -(-total // block_pairs))
    bsz = -(-n // nb)  # query ids per block
    bounds = [min(b * bsz, n) for b in range(nb + 1)]
    bkeys = torch.tensor([lo << 32 for lo in bounds], dtype=torch.int64, device=pairs_dev.device)
    pieces = [[] for _ in range(nb)]
    for s in range(0, total, SLAB):
        sl = pairs_dev[s:s + SLAB]
        key = (sl[:, 0].to(torch.int64) << 32) | (sl[:, 1].to(torch.int64) & 0xFFFFFFFF)
        key = torch.sort(key).values
        cut = torch.searchsorted(key, bkeys).tolist()
        for b in range(nb):
            if cut[b + 1] > cut[b]:
                pieces[b].append(key[cut[b]:cut[b + 1]])
    own = grid is None
    g = oracle.Grid(pts, eps) if own else grid
    try:
        for b in range(nb):
            lo, hi = bounds[b], bounds[b + 1]
            want = g.keys_range(lo, hi)
            if pieces[b]:
                got = torch.sort(torch.cat(pieces[b])).values.cpu().numpy().view(np.uint64)
            else:
                got = np.zeros(0, dtype=np.uint64)
            pieces[b] = None
            if got.shape != want.shape or not np.array_equal(got, want):
                bad = _first_difference(got, want)
                raise AssertionError(f"queries [{lo}, {hi}): {got.shape[0]} GPU pairs vs {want.shape[0]} oracle pairs; "
                                     f"first difference {bad}")
    finally:
        if own:
            g.close()
    return total, nb


def _first_difference(got, want):
    m = min(got.shape[0], want.shape[0])
    d = np.nonzero(got[:m] != want[:m])[0]
    k = int(d[0]) if d.shape[0] else m
    fmt = lambda a: (int(a[k]) >> 32, int(a[k]) & 0xFFFFFFFF) if k < a.shape[0] else None  # noqa: E731
    return {"index": k, "gpu": fmt(got), "oracle": fmt(want)}
