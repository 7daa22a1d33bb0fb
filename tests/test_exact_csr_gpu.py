"""SURVEY §8(f)2 on the GPU: exact two-pass sizing (SJ_OPT_EXACT) and the device-resident CSR
neighbour lists (sj_neighbor_csr), against the oracle.  -m gpu.

Exact sizing must return the oracle's pair set like the estimator path, with no retries, an
exact `est_pairs`, and -- its extra promise -- the same pair ORDER on every run and across the
in-place and staged (host / small-batch / SJ_MORE) deliveries.  The CSR rows must hold, per input
id, exactly the oracle's neighbours (row contents sorted before comparing: the kernel writes
them in neighbourhood traversal order), with row_off the exclusive scan of the oracle degrees.
"""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

import oracle  # noqa: E402
import paper_conf_ipps_galletg19_b200 as sj  # noqa: E402
import workloads  # noqa: E402

DEV = "cuda:0"
CASES = [("c1", None), ("c2k64", 40_009), ("c3k64", 30_011), ("c4k32", 12_007), ("c5", 60_013)]


def points(name, n):
    cfg = workloads.get_config(name)
    if n is not None:
        cfg = cfg.scaled(n)
    return cfg.points(), cfg.eps


def dev(pts):
    return torch.from_numpy(np.ascontiguousarray(pts)).to(DEV)


def join_raw(h, device_out=True, cap=None):
    """All pairs of one join in delivery order (uint32 (M, 2)), via SJ_MORE continuation if cap is small."""
    total = h.count()
    cap = cap or max(total, 1)
    chunks, rc = [], sj.SJ_MORE
    while rc == sj.SJ_MORE:
        if device_out:
            buf = torch.empty((cap, 2), dtype=torch.int32, device=DEV)
        else:
            buf = torch.empty((cap, 2), dtype=torch.int32, pin_memory=True)
        rc, c = h.self_join(buf, cap)
        chunks.append(buf[:c].cpu().numpy().view(np.uint32).copy())
    return np.concatenate(chunks) if chunks else np.zeros((0, 2), np.uint32), total


def csr_want(pts, eps):
    """Oracle CSR: the canonical (sorted) oracle pairs grouped by their first id."""
    pairs = oracle.grid_pairs(pts, eps)
    n = pts.shape[0]
    deg = np.bincount(pairs[:, 0].astype(np.int64), minlength=n)
    off = np.zeros(n + 1, np.int64)
    np.cumsum(deg, out=off[1:])
    return off, pairs[:, 1].astype(np.uint32)


def sort_rows(off, nbrs):
    out = nbrs.copy()
    for i in range(len(off) - 1):
        out[off[i]:off[i + 1]] = np.sort(out[off[i]:off[i + 1]])
    return out


# ------------------------------------------------------------------ exact two-pass sizing

@pytest.mark.parametrize("name,n", CASES)
@pytest.mark.parametrize("pattern", ["lid_unicomp", "gcg", "unicomp"])
def test_exact_matches_oracle_and_is_deterministic(name, n, pattern):
    pts, eps = points(name, n)
    want = oracle.grid_pairs(pts, eps)
    d = dev(pts)
    with sj.Handle(d, eps, pattern=pattern, exact=1) as h:
        a1, total = join_raw(h)
        st = h.stats()
        a2, _ = join_raw(h)
    np.testing.assert_array_equal(oracle.canonical(a1), want)
    assert st["retries"] == 0 and st["est_pairs"] == total == want.shape[0] and st["fast_path"] == 1
    np.testing.assert_array_equal(a1, a2)  # same ORDER on a second run


@pytest.mark.parametrize("name,n", [("c2k64", 40_009), ("c4k32", 12_007), ("c5", 60_013)])
def test_exact_staged_deliveries_keep_the_order(name, n):
    """Staged batches (tiny b_s, host buffer, SJ_MORE with an odd cap) deliver exactly the in-place order."""
    pts, eps = points(name, n)
    d = dev(pts)
    with sj.Handle(d, eps, exact=1) as h:
        ref, total = join_raw(h)
    np.testing.assert_array_equal(oracle.canonical(ref), oracle.grid_pairs(pts, eps))
    for opts, kw in [(dict(fast_path=0), {}), (dict(batch_pairs=20_000), dict(device_out=False)),
                     (dict(batch_pairs=4_096, streams=2), dict(device_out=False, cap=10_007)),
                     (dict(batch_pairs=64, streams=1), dict(cap=total // 3 + 1))]:
        with sj.Handle(d, eps, exact=1, **opts) as h:
            got, _ = join_raw(h, **kw)
            st = h.stats()
        np.testing.assert_array_equal(got, ref, err_msg=str(opts))
        assert st["retries"] == 0
        if opts.get("batch_pairs", 10**8) < total:
            assert st["batches"] > 1


def test_exact_single_chunk_larger_than_batch():
    """A chunk whose pairs exceed b_s gets a batch (and buffer) of its own."""
    rng = np.random.default_rng(7)
    pts = np.concatenate([np.zeros((300, 2)), rng.random((2000, 2)) * 10])  # 300 duplicates: 89700 pairs
    want = oracle.grid_pairs(pts, 0.05)
    with sj.Handle(dev(pts), 0.05, exact=1, batch_pairs=1000, fast_path=0) as h:
        got, _ = join_raw(h, device_out=False)
        st = h.stats()
    np.testing.assert_array_equal(oracle.canonical(got), want)
    assert st["retries"] == 0 and st["batches"] > 1


@pytest.mark.parametrize("k", [1, 2, 4, 16, 32])
def test_exact_other_k(k):
    pts, eps = points("c3k64", 20_011)
    with sj.Handle(dev(pts), eps, exact=1, k=k) as h:
        got, _ = join_raw(h)
    np.testing.assert_array_equal(oracle.canonical(got), oracle.grid_pairs(pts, eps))


@pytest.mark.parametrize("world", [2, 3])
def test_exact_slices_disjoint_union(world):
    pts, eps = points("c5", 40_009)
    d = dev(pts)
    parts = []
    for r in range(world):
        with sj.Handle(d, eps, exact=1) as h:
            h.set_slice(r, world)
            got, _ = join_raw(h)
            parts.append(got)
    np.testing.assert_array_equal(oracle.canonical(np.concatenate(parts)), oracle.grid_pairs(pts, eps))


def test_exact_edge_cases():
    for pts, eps in [(np.zeros((1, 3)), 1.0), (np.arange(10.0).reshape(5, 2), 0.1),
                     (np.zeros((64, 2)), 1.0)]:
        with sj.Handle(dev(pts), eps, exact=1) as h:
            got, total = join_raw(h)
        np.testing.assert_array_equal(oracle.canonical(got), oracle.bf_pairs(pts, eps))


# ------------------------------------------------------------------ device CSR

@pytest.mark.parametrize("name,n", CASES)
@pytest.mark.parametrize("k", [1, 8, 32])
def test_csr_matches_oracle(name, n, k):
    pts, eps = points(name, n)
    off_w, nb_w = csr_want(pts, eps)
    with sj.Handle(dev(pts), eps, pattern="gcg", k=k) as h:
        off, nbrs = h.neighbor_csr(DEV)
        off2, nbrs2 = h.neighbor_csr(DEV)
        st = h.stats()
    off = off.cpu().numpy()
    got = nbrs.cpu().numpy().view(np.uint32)
    np.testing.assert_array_equal(off, off_w)
    np.testing.assert_array_equal(sort_rows(off, got), nb_w)
    np.testing.assert_array_equal(got, nbrs2.cpu().numpy().view(np.uint32))  # deterministic rows
    np.testing.assert_array_equal(off, off2.cpu().numpy())
    assert st["pairs"] == nb_w.shape[0] and st["join_launches"] == 2


def test_csr_host_buffers_and_errors():
    pts, eps = points("c2k64", 30_011)
    off_w, nb_w = csr_want(pts, eps)
    with sj.Handle(dev(pts), eps, pattern="gcg") as h:
        off, nbrs = h.neighbor_csr("cpu")
        np.testing.assert_array_equal(off.numpy(), off_w)
        np.testing.assert_array_equal(sort_rows(off_w, nbrs.numpy().view(np.uint32)), nb_w)
        small = torch.empty(10, dtype=torch.int32, device=DEV)
        row = torch.empty(pts.shape[0] + 1, dtype=torch.int64, device=DEV)
        with pytest.raises(sj.SJError) as e:
            sj.sj_neighbor_csr(h.h, row, small, 10)
        assert e.value.code == sj.SJ_EINVAL
        np.testing.assert_array_equal(row.cpu().numpy(), off_w)  # offsets filled before the error
        # the handle stays usable: the pair join still matches
        got = sj.self_join_pairs(h, DEV).cpu().numpy().view(np.uint32).reshape(-1, 2)
        np.testing.assert_array_equal(oracle.canonical(got), oracle.grid_pairs(pts, eps))
    with sj.Handle(dev(pts), eps) as h:  # LID-UNICOMP handle: rows are not owned by one query
        with pytest.raises(sj.SJError) as e:
            h.neighbor_csr(DEV)
        assert e.value.code == sj.SJ_EINVAL


def test_csr_edge_cases():
    for pts, eps in [(np.zeros((1, 2)), 1.0), (np.arange(12.0).reshape(6, 2), 0.5), (np.zeros((80, 3)), 0.5),
                     (np.random.default_rng(3).random((3000, 6)), 0.3)]:
        off_w, nb_w = csr_want(pts, eps)
        with sj.Handle(dev(pts), eps, pattern="gcg") as h:
            off, nbrs = h.neighbor_csr(DEV)
        off = off.cpu().numpy()
        np.testing.assert_array_equal(off, off_w)
        np.testing.assert_array_equal(sort_rows(off, nbrs.cpu().numpy().view(np.uint32)), nb_w)
