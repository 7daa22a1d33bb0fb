"""Spatially partitioned joins: sj_create_part handles -- own points as
queries, the next slab's first cell column as halo, the global grid origin and global ids --
must return disjoint pair sets whose union is the oracle's.  Single process (slabs cut in
numpy) and the full dist.partitioned_self_join across 2-3 processes sharing cuda:0 (gloo).
-m gpu."""
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

import torch.distributed as dist  # noqa: E402
import torch.multiprocessing as mp  # noqa: E402

import oracle  # noqa: E402
import paper_conf_ipps_galletg19_b200 as sj  # noqa: E402
import workloads  # noqa: E402
from paper_conf_ipps_galletg19_b200 import dist as sjdist  # noqa: E402
from slab_ref import RefRouter, columns_of, owners  # noqa: E402

DEV = "cuda:0"


def cut_slabs(pts, eps, nslab):
    """Slabs of whole dimension-0 cell columns (balanced by points) + the halo of each."""
    origin = pts.min(0)
    col = columns_of(pts[:, 0], float(origin[0]), eps)
    owner_col = owners(np.bincount(col), nslab)
    own = owner_col[col]
    prev = owner_col[np.maximum(col - 1, 0)]
    out = []
    for s in range(nslab):
        mine = np.nonzero(own == s)[0]
        halo = np.nonzero((col >= 1) & (prev != own) & (prev == s))[0]
        ids = np.concatenate([mine, halo]).astype(np.uint32)
        out.append((np.ascontiguousarray(pts[ids]), ids, mine.shape[0]))
    return origin, out


def part_pairs(ppts, ids, nq, eps, origin, ids_on_device=False, **opts):
    if ppts.shape[0] == 0:  # an empty slab (more slabs than occupied cell columns)
        return np.zeros((0, 2), dtype=np.uint32), {"calcs_measured": 0, "dist_calcs": 0}
    d = torch.from_numpy(ppts).to(DEV)
    idt = torch.from_numpy(ids.view(np.int32)).to(DEV) if ids_on_device else ids
    with sj.Handle(d, eps, part=(idt, nq, origin), k=8, count_calcs=1, **opts) as h:
        got = sj.self_join_pairs(h, DEV).cpu().numpy().view(np.uint32).reshape(-1, 2)
        st = h.stats()
    return got, st


@pytest.mark.parametrize("name,n", [("c1", None), ("c2k64", 60_011), ("c3k64", 50_021), ("c5", 80_000),
                                    ("c4k32", 20_011)])
@pytest.mark.parametrize("nslab", [1, 2, 5])
def test_slabs_union_equals_oracle(name, n, nslab):
    cfg = workloads.get_config(name)
    if n is not None:
        cfg = cfg.scaled(n)
    pts = cfg.points()
    want = oracle.grid_pairs(pts, cfg.eps)
    g = oracle.grid_count(pts, cfg.eps, with_hash=False)
    origin, slabs = cut_slabs(pts, cfg.eps, nslab)
    parts, calcs = [], 0
    for i, (ppts, ids, nq) in enumerate(slabs):
        got, st = part_pairs(ppts, ids, nq, cfg.eps, origin, ids_on_device=bool(i % 2))
        assert st["calcs_measured"] == st["dist_calcs"]
        calcs += st["dist_calcs"]
        parts.append(got)
    cat = np.concatenate(parts)
    assert cat.shape == want.shape                      # disjoint partitions
    np.testing.assert_array_equal(oracle.canonical(cat), want)
    assert calcs == g["calcs"] // 2                     # D_alg splits exactly over the slabs


def test_partition_staged_and_exact():
    cfg = workloads.get_config("c5").scaled(60_013)
    pts = cfg.points()
    want = oracle.grid_pairs(pts, cfg.eps)
    origin, slabs = cut_slabs(pts, cfg.eps, 3)
    for opts in ({"fast_path": 0, "batch_pairs": 20_000}, {"exact": 1}, {"queue": 0}):
        cat = np.concatenate([part_pairs(p, i, nq, cfg.eps, origin, **opts)[0] for p, i, nq in slabs])
        np.testing.assert_array_equal(oracle.canonical(cat), want)


def test_partition_errors_and_edges():
    pts = workloads.uniform(5000, 2, 3)
    eps = 0.05
    origin = pts.min(0)
    with pytest.raises(sj.SJError):  # a point below the origin
        sj.Handle(torch.from_numpy(pts).to(DEV), eps, part=(None, 5000, origin + 0.01))
    with pytest.raises(sj.SJError):  # a cell with both query and halo points
        sj.Handle(torch.from_numpy(pts).to(DEV), eps, part=(None, 2500, origin))
    # no queries: nothing to join; ids None: input positions
    with sj.Handle(torch.from_numpy(pts).to(DEV), eps, part=(None, 0, origin)) as h:
        assert h.count() == 0
    with sj.Handle(torch.from_numpy(pts).to(DEV), eps, part=(None, 5000, origin)) as h:
        got = sj.self_join_pairs(h, DEV).cpu().numpy().view(np.uint32).reshape(-1, 2)
    np.testing.assert_array_equal(oracle.canonical(got), oracle.grid_pairs(pts, eps))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, name, n, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        cfg = workloads.get_config(name).scaled(n)
        pts = cfg.points()
        home = np.random.default_rng(5).integers(0, world, pts.shape[0])
        sel = np.nonzero(home == rank)[0]
        pairs, local, total = sjdist.partitioned_self_join(torch.from_numpy(pts[sel]).cuda(),
                                                           torch.from_numpy(sel.astype(np.int32)).cuda(), cfg.eps, k=8)
        q.put((rank, pairs.cpu().numpy().view(np.uint32).reshape(-1, 2).copy(), local, total))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,name,n", [(2, "c5", 80_000), (3, "c3k64", 50_000)])
def test_partitioned_join_across_processes(world, name, n):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, name, n, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict((r[0], r[1:]) for r in (q.get(timeout=300) for _ in range(world)))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    cfg = workloads.get_config(name).scaled(n)
    want = oracle.grid_pairs(cfg.points(), cfg.eps)
    cat = np.concatenate([res[r][0] for r in range(world)])
    assert cat.shape == want.shape
    np.testing.assert_array_equal(oracle.canonical(cat), want)
    for r in range(world):
        assert res[r][2] == want.shape[0] and res[r][1] == res[r][0].shape[0]


# ------------------------------------------------------------------ the slab arithmetic in libsj

def boundary_points(seed=3):
    """Points on, just below and just above dimension-0 column boundaries (x = o + k w (1 + d),
    d in {-2^-52, 0, 2^-52}): where a rounding difference between two column computations would
    put a point in another column than the build's own cell ids."""
    rng = np.random.default_rng(seed)
    eps = 0.013
    w = eps * (1.0 + 2.0 ** -20)
    k = rng.integers(0, 300, 6000).astype(np.float64)
    d = rng.choice([-2.0 ** -52, 0.0, 2.0 ** -52], 6000)
    x0 = 0.25 + k * w * (1.0 + d)
    x0[0] = 0.25  # the origin itself
    x1 = rng.random(6000) * 0.5
    return np.ascontiguousarray(np.stack([x0, x1], 1)), eps


def router_cases():
    out = []
    for name, n in (("c5", 70_001), ("c3k64", 50_021), ("c4k32", 20_011), ("c1", None)):
        cfg = workloads.get_config(name)
        cfg = cfg.scaled(n) if n else cfg
        out.append((name, cfg.points(), cfg.eps))
    pb, eb = boundary_points()
    out.append(("boundaries", pb, eb))
    return out


@pytest.mark.parametrize("name,pts,eps", router_cases(), ids=[c[0] for c in router_cases()])
@pytest.mark.parametrize("world", [1, 2, 3, 8])
def test_lib_router_equals_reference(name, pts, eps, world):
    lib, ref = sjdist.LibRouter(), RefRouter()
    dp = torch.from_numpy(pts).to(DEV)
    cp = torch.from_numpy(pts)
    ids = torch.from_numpy((np.arange(pts.shape[0]) * 7 + 3).astype(np.int32))
    assert lib.bounds(dp) == ref.bounds(cp)
    mn, mx = ref.bounds(cp)
    ncol = lib.columns(mn[0], mx[0], eps)
    assert ncol == ref.columns(mn[0], mx[0], eps)
    h_lib = lib.histogram(dp, mn[0], eps, ncol)
    h_ref = ref.histogram(cp, mn[0], eps, ncol)
    np.testing.assert_array_equal(h_lib.cpu().numpy(), h_ref.numpy())
    # a "global" histogram: this rank's, plus a second rank holding the same points shifted
    got = lib.pack(dp, ids.to(DEV), mn[0], eps, h_lib, world)
    want = ref.pack(cp, ids, mn[0], eps, h_ref, world)
    for g, w_ in zip(got, want):
        if isinstance(w_, list):
            assert g == w_
        else:
            rows = int(w_.shape[0])
            np.testing.assert_array_equal(g[:rows].cpu().numpy(), w_.numpy())


def test_boundary_points_partition_like_the_build():
    """The slab cut by libsj's columns never splits a cell of the build (sj_create_part rejects
    a cell that mixes query and halo points), and the union of the slabs is the oracle's join."""
    pts, eps = boundary_points()
    want = oracle.grid_pairs(pts, eps)
    lib = sjdist.LibRouter()
    dp = torch.from_numpy(pts).to(DEV)
    mn, mx = lib.bounds(dp)
    ncol = lib.columns(mn[0], mx[0], eps)
    hist = lib.histogram(dp, mn[0], eps, ncol)
    world = 5
    own_p, own_i, oc, halo_p, halo_i, hc = lib.pack(dp, None, mn[0], eps, hist, world)
    parts, o0, h0 = [], 0, 0
    for r in range(world):
        p = torch.cat([own_p[o0:o0 + oc[r]], halo_p[h0:h0 + hc[r]]]).contiguous()
        i = torch.cat([own_i[o0:o0 + oc[r]], halo_i[h0:h0 + hc[r]]]).contiguous()
        o0 += oc[r]
        h0 += hc[r]
        if p.shape[0] == 0:
            continue
        with sj.Handle(p, eps, part=(i, oc[r], mn), k=8) as h:
            parts.append(sj.self_join_pairs(h, DEV).cpu().numpy().view(np.uint32).reshape(-1, 2))
    cat = np.concatenate(parts)
    assert cat.shape == want.shape
    np.testing.assert_array_equal(oracle.canonical(cat), want)


def test_router_rejects_bad_input():
    lib = sjdist.LibRouter()
    dp = torch.tensor([[0.0, 1.0], [float("inf"), 2.0]], dtype=torch.float64, device=DEV)
    with pytest.raises(sj.SJError):
        lib.bounds(dp)
    ok = torch.tensor([[0.0, 1.0], [3.0, 2.0]], dtype=torch.float64, device=DEV)
    with pytest.raises(sj.SJError):  # a point beyond the last column
        lib.histogram(ok, 0.0, 1.0, 2)
    with pytest.raises(sj.SJError):  # below the origin
        lib.histogram(ok, 1.0, 1.0, 8)
    with pytest.raises(sj.SJError):
        lib.columns(0.0, 1e12, 1e-6)  # >= 2^30 columns
