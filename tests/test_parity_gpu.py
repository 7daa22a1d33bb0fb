"""Parity of the CUDA path (through the C ABI) against the CPU oracle.  -m gpu.

Bar (BASELINE.json north_star): the GPU pair SET is bit-exact against
the oracle after canonical (i, j) sorting -- integer/index output, both sides with
FP64 RN dimension-order accumulation, no FMA, s <= fl(eps^2).  Every size is compared
element by element (full BASELINE sizes in tests/test_fullsize_gpu.py).
"""
import math
import os

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

import oracle  # noqa: E402
import paper_conf_ipps_galletg19_b200 as sj  # noqa: E402
import workloads  # noqa: E402
from conftest import load_golden  # noqa: E402

DEV = "cuda:0"


def gpu_pairs(pts, eps, k=8, device_out=True, points_on_device=True, **opts):
    p = torch.from_numpy(np.ascontiguousarray(pts)).to(DEV) if points_on_device else np.ascontiguousarray(pts)
    with sj.Handle(p, eps, k=k, **opts) as h:
        out = sj.self_join_pairs(h, DEV if device_out else "cpu")
        st = h.stats()
    a = out.cpu().numpy().view(np.uint32).reshape(-1, 2)
    return a, st


def canon(a):
    return oracle.canonical(a)


# ------------------------------------------------------------------ worked examples

@pytest.mark.parametrize("name", ["tiny_2d.txt", "tiny_3d.txt"])
@pytest.mark.parametrize("k", [1, 8, 32])
def test_golden(name, k):
    pts, eps, expected = load_golden(name)
    got, _ = gpu_pairs(pts, eps, k=k)
    np.testing.assert_array_equal(canon(got), canon(expected))


# ------------------------------------------------------------------ C1 element by element vs O1

@pytest.mark.parametrize("k", [1, 2, 4, 8, 16, 32])
def test_c1_bruteforce_all_k(k):
    cfg = workloads.get_config("c1")
    pts = cfg.points()
    want = oracle.bf_pairs(pts, cfg.eps)
    got, st = gpu_pairs(pts, cfg.eps, k=k, count_calcs=1)
    np.testing.assert_array_equal(canon(got), want)
    # kernel accounting: instrumented calcs == D_alg (a7) == half the oracle's full 3^n scan
    g = oracle.grid_count(pts, cfg.eps, with_hash=False)
    assert st["calcs_measured"] == st["dist_calcs"] == g["calcs"] // 2
    assert g["calcs"] % 2 == 0
    assert st["n_cells"] == g["ncells"]


# ------------------------------------------------------------------ mid sizes vs O2 element by element

MID = [("c2k64", 150_001), ("c2k16", 120_007), ("c3k64", 150_013), ("c4k32", 60_017), ("c5", 200_003),
       ("c2k256", 60_001), ("c3k256", 80_021)]


@pytest.mark.parametrize("name,n", MID)
def test_mid_size_elementwise(name, n):
    cfg = workloads.get_config(name).scaled(n)
    pts = cfg.points()
    want = oracle.grid_pairs(pts, cfg.eps)
    got, st = gpu_pairs(pts, cfg.eps, k=cfg.k, count_calcs=1)
    assert got.shape == want.shape, (got.shape, want.shape)
    np.testing.assert_array_equal(canon(got), want)
    g = oracle.grid_count(pts, cfg.eps, with_hash=False)
    assert st["calcs_measured"] == st["dist_calcs"] == g["calcs"] // 2


@pytest.mark.parametrize("k", [1, 4, 32])
@pytest.mark.parametrize("name", ["c3k64", "c4k32"])
def test_mid_size_other_k(name, k):
    cfg = workloads.get_config(name).scaled(40_009)
    pts = cfg.points()
    want = oracle.grid_pairs(pts, cfg.eps)
    got, _ = gpu_pairs(pts, cfg.eps, k=k)
    np.testing.assert_array_equal(canon(got), want)


@pytest.mark.parametrize("dim", [1, 2, 3, 4, 5, 6, 7, 8])
def test_every_dimension(dim):
    n = 20_000 if dim <= 4 else 6_000
    pts = workloads.uniform(n, dim, 300 + dim)
    eps = workloads.eps_for_k("uniform", n, dim, 12)
    want = oracle.grid_pairs(pts, eps)
    got, _ = gpu_pairs(pts, eps, k=4)
    np.testing.assert_array_equal(canon(got), want)


# ------------------------------------------------------------------ batching, overflow, continuation

def test_staged_batches_and_overflow_retry():
    cfg = workloads.get_config("c3k64").scaled(100_003)
    pts = cfg.points()
    want = oracle.grid_pairs(pts, cfg.eps)
    # tiny b_s forces many batches; a tiny estimator sample forces underestimates -> overflow retries
    got, st = gpu_pairs(pts, cfg.eps, k=8, batch_pairs=20_000, sample_ppm=1, fast_path=0, streams=3)
    np.testing.assert_array_equal(canon(got), want)
    assert st["batches"] > 5
    got2, st2 = gpu_pairs(pts, cfg.eps, k=8, batch_pairs=7_000, fast_path=0, streams=2, sample_ppm=100)
    np.testing.assert_array_equal(canon(got2), want)


def test_sj_more_continuation_host_buffer():
    cfg = workloads.get_config("c5").scaled(50_000)
    pts = cfg.points()
    want = oracle.grid_pairs(pts, cfg.eps)
    p = torch.from_numpy(pts).to(DEV)
    with sj.Handle(p, cfg.eps, k=8, batch_pairs=30_000) as h:
        cap = 12_345
        buf = np.empty((cap, 2), dtype=np.uint32)  # pageable host memory
        parts, rc, calls = [], sj.SJ_MORE, 0
        while rc == sj.SJ_MORE:
            rc, c = h.self_join(buf, cap)
            parts.append(buf[:c].copy())
            calls += 1
            assert calls < 10_000
        got = np.concatenate(parts)
        assert calls > 3
        # a new call after SJ_OK restarts the join and yields the same set
        rc, c = h.self_join(buf, cap)
        assert rc in (sj.SJ_OK, sj.SJ_MORE)
    np.testing.assert_array_equal(canon(got), want)


def test_device_buffer_too_small_falls_back_to_continuation():
    cfg = workloads.get_config("c2k64").scaled(40_000)
    pts = cfg.points()
    want = oracle.grid_pairs(pts, cfg.eps)
    p = torch.from_numpy(pts).to(DEV)
    with sj.Handle(p, cfg.eps, k=8) as h:
        cap = want.shape[0] // 3 + 1
        buf = torch.empty((cap, 2), dtype=torch.int32, device=DEV)
        parts, rc = [], sj.SJ_MORE
        while rc == sj.SJ_MORE:
            rc, c = h.self_join(buf, cap)
            parts.append(buf[:c].cpu().numpy().view(np.uint32).copy())
    np.testing.assert_array_equal(canon(np.concatenate(parts)), want)


@pytest.mark.parametrize("device_out,points_on_device", [(False, False), (True, False), (False, True)])
def test_host_and_device_pointers(device_out, points_on_device):
    cfg = workloads.get_config("c1")
    pts = cfg.points()
    want = oracle.bf_pairs(pts, cfg.eps)
    got, _ = gpu_pairs(pts, cfg.eps, k=8, device_out=device_out, points_on_device=points_on_device)
    np.testing.assert_array_equal(canon(got), want)


def test_misaligned_device_input_and_odd_sizes():
    # a device pointer 8 bytes into an allocation (not 16-byte aligned) and an odd number of
    # coordinates (3-D, odd n) exercise the bbox reader's edge cases
    for dim, n in ((3, 10_001), (1, 9_999), (5, 3_333)):
        pts = workloads.uniform(n, dim, 900 + dim)
        eps = workloads.eps_for_k("uniform", n, dim, 10)
        big = torch.empty(n * dim + 1, dtype=torch.float64, device=DEV)
        big[1:] = torch.from_numpy(pts.ravel()).to(DEV)
        view = big[1:].view(n, dim)
        assert view.data_ptr() % 16 == 8
        with sj.Handle(view, eps, k=8) as h:
            got = sj.self_join_pairs(h, DEV).cpu().numpy().view(np.uint32)
        np.testing.assert_array_equal(canon(got), oracle.grid_pairs(pts, eps))


def test_count_only_matches_oracle():
    cfg = workloads.get_config("c3k64").scaled(100_000)
    pts = cfg.points()
    with sj.Handle(torch.from_numpy(pts).to(DEV), cfg.eps) as h:
        assert h.count() == oracle.grid_count(pts, cfg.eps, with_hash=False)["count"]


# ------------------------------------------------------------------ edge cases

def test_single_point():
    got, st = gpu_pairs(np.array([[0.5, 0.5]]), 0.1)
    assert got.shape[0] == 0 and st["n_cells"] == 1


def test_all_duplicates():
    n = 3000
    got, _ = gpu_pairs(workloads.duplicates(n, 3), 1e-6, k=8)
    assert got.shape[0] == n * (n - 1)
    np.testing.assert_array_equal(canon(got), oracle.bf_pairs(workloads.duplicates(n, 3), 1e-6))


def test_one_cell_huge_eps():
    pts = workloads.uniform(2000, 2, 4)
    got, st = gpu_pairs(pts, 10.0, k=32)
    assert got.shape[0] == 2000 * 1999 and st["n_cells"] == 1


def test_eps_below_spacing_is_empty():
    got, _ = gpu_pairs(workloads.lattice(30, 2), 0.999)
    assert got.shape[0] == 0


@pytest.mark.parametrize("dim,g", [(2, 60), (3, 20), (6, 5)])
def test_lattice_closed_form(dim, g):
    got, _ = gpu_pairs(workloads.lattice(g, dim), 1.0, k=8)
    assert got.shape[0] == 2 * dim * g ** (dim - 1) * (g - 1)


def test_ragged_tail_and_grab_sizes():
    cfg = workloads.get_config("c2k32").scaled(33_333)
    pts = cfg.points()
    want = oracle.grid_pairs(pts, cfg.eps)
    for grab in (4, 8, 40, 1024):
        got, _ = gpu_pairs(pts, cfg.eps, k=8, grab=grab)
        np.testing.assert_array_equal(canon(got), want)


def test_invalid_inputs():
    with pytest.raises(sj.SJError, match="non-finite"):
        sj.Handle(torch.tensor([[0.0, 1.0], [float("nan"), 2.0]], dtype=torch.float64, device=DEV), 0.5)
    with pytest.raises(sj.SJError, match="grid too large"):
        sj.Handle(np.array([[0.0, 0.0], [1e12, 0.0]]), 1e-6)
    with sj.Handle(np.zeros((3, 2)), 1.0) as h:
        with pytest.raises(sj.SJError):
            h.self_join(None, 5)


# ------------------------------------------------------------------ multi-GPU slices (sequential, one GPU)

@pytest.mark.parametrize("world", [2, 3, 8])
def test_slices_disjoint_union(world):
    cfg = workloads.get_config("c5").scaled(60_000)
    pts = cfg.points()
    want = oracle.grid_pairs(pts, cfg.eps)
    p = torch.from_numpy(pts).to(DEV)
    parts = []
    with sj.Handle(p, cfg.eps, k=8) as h:
        for r in range(world):
            h.set_slice(r, world)
            parts.append(sj.self_join_pairs(h, DEV).cpu().numpy().view(np.uint32))
    cat = np.concatenate(parts)
    assert cat.shape == want.shape  # disjoint: no pair evaluated twice
    np.testing.assert_array_equal(canon(cat), want)


def test_index_blob_roundtrip():
    cfg = workloads.get_config("c3k64").scaled(50_000)
    pts = cfg.points()
    want = oracle.grid_pairs(pts, cfg.eps)
    with sj.Handle(torch.from_numpy(pts).to(DEV), cfg.eps) as h:
        nbytes = h.export_index()
        blob = torch.empty(nbytes, dtype=torch.uint8, device=DEV)
        h.export_index(blob, nbytes)
        host_blob = blob.cpu().numpy()
    with sj.Handle.from_index(blob, nbytes) as h2:
        got = sj.self_join_pairs(h2, DEV).cpu().numpy().view(np.uint32)
    np.testing.assert_array_equal(canon(got), want)
    with sj.Handle.from_index(host_blob, nbytes) as h3:
        assert h3.count() == want.shape[0]
    # zero-copy view of a device blob: the handle's arrays are the blob's
    with sj.Handle.from_index(blob, nbytes, view=True) as h4:
        got4 = sj.self_join_pairs(h4, DEV).cpu().numpy().view(np.uint32)
    np.testing.assert_array_equal(canon(got4), want)
    with pytest.raises(sj.SJError):  # a host blob cannot be viewed
        sj.Handle.from_index(host_blob, nbytes, view=True)

# (full BASELINE sizes: tests/test_fullsize_gpu.py, element by element)


# ------------------------------------------------------------------ blocked in-place output

@pytest.mark.parametrize("name,n", [("c2k64", 150_001), ("c3k64", 150_013), ("c5", 200_003), ("c4k32", 40_009)])
@pytest.mark.parametrize("slack", [0, 1, 777_777])
def test_blocked_output_elementwise(name, n, slack):
    """SJ_OPT_OUT_BLOCKS=1: every warp takes output blocks of 4096 pairs (one atomic per block);
    the warps' last blocks leave gaps that the compaction pass closes, positions past the caller's
    buffer go to the scratch and are moved back.  Exactly sized, odd-sized (+1) and large buffers."""
    cfg = workloads.get_config(name).scaled(n)
    pts = cfg.points()
    want = oracle.grid_pairs(pts, cfg.eps)
    p = torch.from_numpy(pts).to(DEV)
    cap = want.shape[0] + slack
    out = torch.full((cap, 2), -1, dtype=torch.int32, device=DEV)
    with sj.Handle(p, cfg.eps, k=cfg.k, out_blocks=1, count_calcs=1) as h:
        rc, c = h.self_join(out, cap)
        st = h.stats()
    assert rc == sj.SJ_OK and c == want.shape[0] and st["fast_path"] == 1
    got = out[:c].cpu().numpy().view(np.uint32)
    np.testing.assert_array_equal(canon(got), want)
    assert st["calcs_measured"] == st["dist_calcs"]


def test_blocked_output_overflow_falls_back():
    cfg = workloads.get_config("c5").scaled(120_007)
    pts = cfg.points()
    want = oracle.grid_pairs(pts, cfg.eps)
    p = torch.from_numpy(pts).to(DEV)
    cap = want.shape[0] // 2 + 1
    with sj.Handle(p, cfg.eps, k=8, out_blocks=1) as h:
        buf = torch.empty((cap, 2), dtype=torch.int32, device=DEV)
        parts, rc = [], sj.SJ_MORE
        while rc == sj.SJ_MORE:
            rc, c = h.self_join(buf, cap)
            parts.append(buf[:c].cpu().numpy().view(np.uint32).copy())
    np.testing.assert_array_equal(canon(np.concatenate(parts)), want)
