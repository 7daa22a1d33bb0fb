"""Spatial slab partitioning (dist.slab_partition) on CPU with gloo, world 2
and 3: the ranks own slabs of whole cell columns along dimension 0 and receive the first
column of the next slab as a halo.  Pinned here, independently of the GPU: every point is
owned by exactly one rank, the slabs are disjoint column ranges balanced by points, the halo
holds exactly the points the LID-UNICOMP pattern (Alg. 3: forward cells are at most
one column ahead) needs, and every oracle pair is visible on the rank owning its lower-column
point.  The GPU join over the partitions is tests/test_partition_gpu.py."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _data(name):
    import workloads

    if name == "c1":
        cfg = workloads.get_config("c1")
    else:
        cfg = workloads.get_config(name).scaled(30_000)
    return cfg.points(), cfg.eps


def _worker(rank, world, port, name, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_ipps_galletg19_b200 import dist as sjdist
        from slab_ref import RefRouter

        pts, eps = _data(name)
        # the input is spread over the ranks arbitrarily (not by space)
        home = np.random.default_rng(11).integers(0, world, pts.shape[0])
        sel = np.nonzero(home == rank)[0]
        p, i, nq, origin = sjdist.slab_partition(torch.from_numpy(pts[sel]), torch.from_numpy(sel.astype(np.int32)),
                                                 eps, router=RefRouter())
        q.put((rank, p.numpy(), i.numpy(), nq, origin))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
@pytest.mark.parametrize("name", ["c1", "c5", "c3k64"])
def test_slab_partition(world, name):
    import oracle
    from slab_ref import columns_of

    ctx = mp.get_context("spawn")
    qq = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, name, qq)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict((r[0], r[1:]) for r in (qq.get(timeout=180) for _ in range(world)))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    pts, eps = _data(name)
    n = pts.shape[0]
    origin = pts.min(0)
    col = columns_of(pts[:, 0], float(origin[0]), eps)
    owner_of = np.full(n, -1)
    local = []
    for r in range(world):
        p, ids, nq, org = res[r]
        assert np.array_equal(np.asarray(org), origin)          # the global origin everywhere
        np.testing.assert_array_equal(p, pts[ids])              # rows travel with their ids
        own = ids[:nq]
        assert np.all(owner_of[own] == -1)                      # owned once
        owner_of[own] = r
        local.append(set(ids.tolist()))
        halo = ids[nq:]
        if nq and halo.size:                                    # halo = next column(s) only
            assert col[halo].min() > col[own].max()
    assert np.all(owner_of >= 0)                                # every point owned
    # slabs: disjoint, ordered column ranges; balanced by points to within a column per cut
    rng = [(col[owner_of == r].min(), col[owner_of == r].max()) for r in range(world) if np.any(owner_of == r)]
    for a, b in zip(rng, rng[1:]):
        assert a[1] < b[0]
    sizes = np.bincount(owner_of, minlength=world)
    assert sizes.max() - sizes.min() <= 2 * np.bincount(col).max() + 1  # a column each side of a cut
    # every oracle pair is visible on the rank owning its lower-column point
    pairs = oracle.grid_pairs(pts, eps)
    lo = np.where(col[pairs[:, 0]] <= col[pairs[:, 1]], pairs[:, 0], pairs[:, 1])
    hi = np.where(col[pairs[:, 0]] <= col[pairs[:, 1]], pairs[:, 1], pairs[:, 0])
    for r in range(world):
        m = owner_of[lo] == r
        assert set(hi[m].tolist()) <= local[r]
