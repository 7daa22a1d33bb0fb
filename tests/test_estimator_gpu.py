"""The batch estimator (a9: "we sample the first 1% of D'") fused into the in-place
join (DESIGN.md §5 "Fast-path estimator").  -m gpu.

The fused counter must return exactly the number a separate count-only launch over the same
sample chunks returns (the staged path, host output, still runs that launch), so the estimate
and the batch count derived from it are unchanged; when the output overflows before the
sample was handed out, the separate launch runs instead.
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


def _estimate(pts, eps, k, device_out, cap=None, **opts):
    d = torch.from_numpy(np.ascontiguousarray(pts)).to(DEV)
    with sj.Handle(d, eps, k=k, **opts) as h:
        total = h.count()
        n = max(total, 1) if cap is None else cap
        if device_out:
            out = torch.empty((n, 2), dtype=torch.int32, device=DEV)
        else:
            out = torch.empty((n, 2), dtype=torch.int32, pin_memory=True)
        rc, got = h.self_join(out, n)
        st = h.stats()
    return st, total, got


@pytest.mark.parametrize("name,n", [("c5", 200_003), ("c3k64", 150_013), ("c2k64", 150_001), ("c4k32", 60_017)])
@pytest.mark.parametrize("ppm", [10_000, 100_000])
def test_fused_estimate_equals_separate(name, n, ppm):
    cfg = workloads.get_config(name).scaled(n)
    pts = cfg.points()
    fused, total, got = _estimate(pts, cfg.eps, cfg.k, True, sample_ppm=ppm)
    sep, total2, _ = _estimate(pts, cfg.eps, cfg.k, False, sample_ppm=ppm)
    assert fused["fast_path"] == 1 and fused["est_fused"] == 1 and fused["ms_estimate"] == 0.0
    assert sep["est_fused"] == 0
    assert fused["est_pairs"] == sep["est_pairs"] > 0
    assert got == total == total2 == oracle.grid_count(pts, cfg.eps, with_hash=False)["count"]


def test_fused_estimate_whole_queue_is_exact():
    # a 100 % sample: the estimate is the exact pair count
    cfg = workloads.get_config("c3k64").scaled(80_021)
    pts = cfg.points()
    st, total, got = _estimate(pts, cfg.eps, 8, True, sample_ppm=1_000_000)
    assert st["est_fused"] == 1 and st["est_pairs"] == total == got


def test_overflow_before_sample_falls_back():
    # a tiny device buffer: the join stops dequeuing after its first flush, before the sample
    # chunks were all handed out -> the separate estimator runs; the estimate is unchanged
    cfg = workloads.get_config("c5").scaled(200_003)
    pts = cfg.points()
    ref, _, _ = _estimate(pts, cfg.eps, 8, False, sample_ppm=100_000)
    st, total, got = _estimate(pts, cfg.eps, 8, True, cap=64, sample_ppm=100_000)
    assert got == 64
    assert st["est_pairs"] == ref["est_pairs"]


# ------------------------------------------------------------------ the lazy build tail
# sj_create returns without a final host round trip; an in-place join issued right after it is
# sized on the device (the kernel reads the build's chunk count).  These tests make the join the
# FIRST call after sj_create (no count() before it), which is the path bench.py times.

def _first_call_join(pts, eps, k=8, cap=None, slice_=None, **opts):
    d = torch.from_numpy(np.ascontiguousarray(pts)).to(DEV)
    n = cap if cap is not None else oracle.grid_count(pts, eps, with_hash=False)["count"]
    out = torch.empty((max(n, 1), 2), dtype=torch.int32, device=DEV)
    with sj.Handle(d, eps, k=k, **opts) as h:
        if slice_:
            h.set_slice(*slice_)
        rc, got = h.self_join(out, max(n, 1))
        st = h.stats()
        total = h.count()  # a second call: the synchronous paths, same handle
        st2 = h.stats()
    return out[:got].cpu().numpy().view(np.uint32).reshape(-1, 2), rc, st, total, st2


@pytest.mark.parametrize("name,n", [("c5", 200_003), ("c3k64", 150_013), ("c4k32", 60_017), ("c1", None)])
def test_lazy_first_join_matches_oracle(name, n):
    cfg = workloads.get_config(name)
    if n:
        cfg = cfg.scaled(n)
    pts = cfg.points()
    got, rc, st, total, st2 = _first_call_join(pts, cfg.eps, k=cfg.k)
    want = oracle.grid_pairs(pts, cfg.eps)
    np.testing.assert_array_equal(oracle.canonical(got), want)
    assert rc == 0 and st["fast_path"] == 1 and st["est_fused"] == 1 and total == want.shape[0]
    # the build's tail reached the host: the static statistics agree with the synchronous read
    for key in ("n_chunks", "fwd_runs", "n_cells", "dist_calcs", "key_bits", "max_cell_load"):
        assert st[key] == st2[key], key
    assert st["n_chunks"] > 0 and st["ms_build"] > 0.0
    # the estimate equals a separate count-only estimator on a handle whose first call was count()
    sep, _, _ = _estimate(pts, cfg.eps, cfg.k, False)
    assert st["est_pairs"] == sep["est_pairs"]


@pytest.mark.parametrize("world", [2, 3])
def test_lazy_first_join_slices(world):
    cfg = workloads.get_config("c3k64").scaled(150_013)
    pts = cfg.points()
    want = oracle.grid_pairs(pts, cfg.eps)
    parts = []
    for r in range(world):
        got, rc, st, total, _ = _first_call_join(pts, cfg.eps, cap=want.shape[0], slice_=(r, world))
        assert rc == 0 and st["est_fused"] == 1 and got.shape[0] == total
        parts.append(got)
    allp = np.concatenate(parts)
    np.testing.assert_array_equal(oracle.canonical(allp), want)


def test_lazy_first_join_overflow():
    cfg = workloads.get_config("c5").scaled(200_003)
    pts = cfg.points()
    ref, _, _ = _estimate(pts, cfg.eps, 8, False, sample_ppm=100_000)
    got, rc, st, total, _ = _first_call_join(pts, cfg.eps, cap=64, sample_ppm=100_000)
    assert rc == 1 and got.shape[0] == 64  # SJ_MORE
    assert st["est_pairs"] == ref["est_pairs"]


def test_points_reusable_when_create_returns():
    # sj_create may return before the build's last kernels ran (lazy tail), but never before the
    # last read of the caller's points: overwriting them right away must not change the result
    cfg = workloads.get_config("c5").scaled(200_003)
    pts = cfg.points()
    want = oracle.grid_pairs(pts, cfg.eps)
    d = torch.from_numpy(np.ascontiguousarray(pts)).to(DEV)
    out = torch.empty((want.shape[0], 2), dtype=torch.int32, device=DEV)
    for _ in range(2):
        d.copy_(torch.from_numpy(pts))
        torch.cuda.synchronize()
        with sj.Handle(d, cfg.eps, k=8) as h:
            d.fill_(float("nan"))  # torch's stream, right after sj_create returned
            rc, got = h.self_join(out, want.shape[0])
        assert rc == 0 and got == want.shape[0]
        np.testing.assert_array_equal(oracle.canonical(out.cpu().numpy().view(np.uint32).reshape(-1, 2)), want)
