"""Reference slab router (test infrastructure): the slab rule of DESIGN.md §6 written out in
numpy on CPU tensors, with the same interface as dist.LibRouter (libsj's sj_part_*).  The CPU
gloo tests drive dist.slab_partition's collective plumbing with it; the GPU tests compare
libsj's router with it call by call.

  column  c = floor(fl(fl(x_0 - origin_0) / w)), w = eps (1 + 2^-20)   (numpy binary64, RN)
  owner   of column c = min(world - 1, floor(start_c * world / total)), start_c = points before c
  halo    points of column c >= 1 with owner(c - 1) != owner(c), sent to owner(c - 1)
Rows grouped by destination rank ascending, input order inside a rank.
"""
from __future__ import annotations

import numpy as np
import torch


def columns_of(x0: np.ndarray, origin0: float, eps: float) -> np.ndarray:
    w = float(eps) * (1.0 + 2.0 ** -20)
    return np.floor((x0 - origin0) / w).astype(np.int64)


def owners(hist: np.ndarray, world: int) -> np.ndarray:
    hist = hist.astype(np.int64)
    total = int(hist.sum())
    if total == 0:
        return np.zeros_like(hist)
    start = np.cumsum(hist) - hist
    return np.minimum((start * world) // total, world - 1)


class RefRouter:
    def bounds(self, points):
        p = points.cpu().numpy()
        if p.shape[0] == 0:
            return [float("inf")] * p.shape[1], [float("-inf")] * p.shape[1]
        return p.min(0).tolist(), p.max(0).tolist()

    def columns(self, origin0, max0, eps):
        return int(columns_of(np.array([max0]), origin0, eps)[0]) + 1

    def histogram(self, points, origin0, eps, ncol):
        col = columns_of(points[:, 0].cpu().numpy(), origin0, eps)
        assert col.size == 0 or (col.min() >= 0 and col.max() < ncol)
        return torch.from_numpy(np.bincount(col, minlength=ncol).astype(np.int64)).to(points.device)

    def pack(self, points, ids, origin0, eps, hist, world):
        p = points.cpu().numpy()
        n = p.shape[0]
        i = ids.cpu().numpy() if ids is not None else np.arange(n, dtype=np.int32)
        col = columns_of(p[:, 0], origin0, eps)
        own_of = owners(hist.cpu().numpy(), world)
        own = own_of[col] if n else np.zeros(0, dtype=np.int64)
        prev = own_of[np.maximum(col - 1, 0)] if n else np.zeros(0, dtype=np.int64)
        halo = (col >= 1) & (prev != own)
        o = np.argsort(own, kind="stable")
        hsel = np.nonzero(halo)[0]
        ho = hsel[np.argsort(prev[hsel], kind="stable")]
        dev = points.device
        t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).to(dev)  # noqa: E731
        return (t(p[o]), t(i[o].astype(np.int32)), np.bincount(own, minlength=world).tolist(),
                t(p[ho]), t(i[ho].astype(np.int32)), np.bincount(prev[hsel], minlength=world).tolist())
