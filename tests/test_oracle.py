"""Pins for the CPU oracle (oracle/) against things other than itself.

Every test here runs on CPU (-m "not gpu").  The oracle must be right before it can
judge the CUDA path, so each function is pinned by something independent:

* hand-computed worked examples (tests/golden/, cited to PAPER.md:44-46);
* closed forms on integer lattices (distances exactly 1, sqrt 2, sqrt 3);
* degenerate cases: all duplicates -> N(N-1); eps below the spacing -> 0;
* a 1-D special case that reduces to sort + binary search (textbook);
* scipy's cKDTree.query_pairs (a library routine) on random 2..6-D data;
* O2 (grid) == O1 (brute force) element by element on small inputs of every
  distribution and dimensionality, with an eps sweep (one cell ... below spacing);
* invariants: symmetric, irreflexive, eps-monotone; count with == without index;
* the grid's neighbourhood guarantee (every O1 pair lies in adjacent cells).
A dropped term, wrong sign/index, transposed operand or exclusive "<" would fail
at least one of these.
"""
import math

import numpy as np
import pytest

import oracle
import workloads
from conftest import load_golden


def _set(pairs):
    a = np.asarray(pairs, dtype=np.uint64).reshape(-1, 2)
    return set(((a[:, 0] << np.uint64(32)) | a[:, 1]).tolist())


# ----------------------------------------------------------------- golden pins

@pytest.mark.parametrize("name", ["tiny_2d.txt", "tiny_3d.txt"])
def test_golden_worked_examples(name):
    pts, eps, expected = load_golden(name)
    exp = oracle.canonical(expected)
    np.testing.assert_array_equal(oracle.bf_pairs(pts, eps), exp)
    np.testing.assert_array_equal(oracle.grid_pairs(pts, eps), exp)
    cnt, h = oracle.bf_count(pts, eps)
    assert cnt == exp.shape[0]
    assert h == oracle.hash_pairs(exp)
    g = oracle.grid_count(pts, eps)
    assert g["count"] == exp.shape[0] and g["hash"] == h


def test_inclusive_boundary_is_exact():
    # dist == eps exactly must be included ("<="); the next double above is not.
    p = np.array([[0.0, 0.0], [0.25, 0.0]])
    assert oracle.bf_count(p, 0.25)[0] == 2
    assert oracle.bf_count(p, np.nextafter(0.25, 0.0))[0] == 0


# ----------------------------------------------------------------- closed forms

@pytest.mark.parametrize("dim,g", [(1, 17), (2, 9), (3, 6), (4, 4), (5, 3), (6, 3)])
def test_lattice_eps1_closed_form(dim, g):
    # g^dim integer lattice, eps = 1: only axis neighbours (distance exactly 1).
    # ordered pairs = 2 * dim * g^(dim-1) * (g-1)
    p = workloads.lattice(g, dim)
    want = 2 * dim * g ** (dim - 1) * (g - 1)
    assert oracle.bf_count(p, 1.0)[0] == want
    assert oracle.grid_count(p, 1.0)["count"] == want


@pytest.mark.parametrize("g", [2, 5, 11])
def test_lattice_2d_eps15_closed_form(g):
    # + diagonals (distance sqrt 2): 4 g (g-1) + 4 (g-1)^2
    p = workloads.lattice(g, 2)
    want = 4 * g * (g - 1) + 4 * (g - 1) ** 2
    assert oracle.bf_count(p, 1.5)[0] == want
    assert oracle.grid_count(p, 1.5)["count"] == want


@pytest.mark.parametrize("g", [2, 4, 7])
def test_lattice_3d_eps15_closed_form(g):
    # axis (1) + face diagonals (sqrt 2); body diagonals (sqrt 3 > 1.5) excluded:
    # 6 g^2 (g-1) + 12 g (g-1)^2
    p = workloads.lattice(g, 3)
    want = 6 * g * g * (g - 1) + 12 * g * (g - 1) ** 2
    assert oracle.bf_count(p, 1.5)[0] == want
    assert oracle.grid_count(p, 1.5)["count"] == want


def test_lattice_spacing_scaled():
    # a non-integer spacing: lattice spacing 0.1 with eps = 0.15 -> axis pairs only
    # (0.1*sqrt2 = 0.1414 < 0.15 -> diagonals too in 2-D).
    g = 8
    p = workloads.lattice(g, 2, spacing=0.1)
    want = 4 * g * (g - 1) + 4 * (g - 1) ** 2
    assert oracle.bf_count(p, 0.15)[0] == want
    assert oracle.grid_count(p, 0.15)["count"] == want


@pytest.mark.parametrize("dim", [1, 2, 3, 6])
def test_all_duplicates(dim):
    n = 57
    p = workloads.duplicates(n, dim)
    assert oracle.bf_count(p, 1e-9)[0] == n * (n - 1)
    g = oracle.grid_count(p, 1e-9)
    assert g["count"] == n * (n - 1) and g["ncells"] == 1


def test_eps_below_spacing_is_empty():
    p = workloads.lattice(6, 3)
    assert oracle.bf_count(p, 0.999)[0] == 0
    assert oracle.grid_count(p, 0.999)["count"] == 0


def test_single_point_and_empty():
    assert oracle.bf_count(np.zeros((1, 3)), 1.0)[0] == 0
    assert oracle.grid_count(np.zeros((1, 3)), 1.0)["count"] == 0
    assert oracle.bf_pairs(np.zeros((0, 2)), 1.0).shape == (0, 2)


# ----------------------------------------------------------------- textbook / library

@pytest.mark.parametrize("seed", [0, 1])
def test_1d_sort_and_search(seed):
    # 1-D: the eps-neighbourhood of x in sorted order is the window [x-eps, x+eps].
    x = np.random.default_rng(seed).random(4000)
    eps = 3e-3
    xs = np.sort(x)
    # guard: no pair sits within 1e-12 of the boundary, so |t| <= eps <=> t^2 <= eps^2
    d = np.abs(xs[None, :200] - xs[:, None])
    assert np.min(np.abs(d - eps)) > 1e-12
    hi = np.searchsorted(xs, xs + eps, side="right")
    lo = np.searchsorted(xs, xs - eps, side="left")
    want = int(np.sum(hi - lo - 1))
    p = x.reshape(-1, 1)
    assert oracle.bf_count(p, eps)[0] == want
    assert oracle.grid_count(p, eps)["count"] == want


@pytest.mark.parametrize("dim,n,k", [(2, 3000, 20), (3, 3000, 20), (4, 2000, 15), (6, 1500, 10)])
def test_matches_scipy_kdtree(dim, n, k):
    from scipy.spatial import cKDTree

    p = workloads.uniform(n, dim, 100 + dim)
    eps = workloads.eps_for_k("uniform", n, dim, k)
    und = cKDTree(p).query_pairs(eps, output_type="ndarray")
    want = set()
    for i, j in und.tolist():
        want.add((i << 32) | j)
        want.add((j << 32) | i)
    got = _set(oracle.grid_pairs(p, eps))
    # scipy compares sqrt-free distances with its own rounding; exclude near-boundary pairs
    diff = got ^ want
    for key in diff:
        i, j = key >> 32, key & 0xFFFFFFFF
        s = float(np.sum((p[i] - p[j]) ** 2))
        assert abs(s - eps * eps) <= 1e-12 * eps * eps, (i, j, s, eps * eps)
    assert len(got) > 0


# ----------------------------------------------------------------- O2 == O1

CASES = []
for dist in ("uniform", "exponential"):
    for dim in (1, 2, 3, 4, 5, 6):
        for k in (0.5, 8, 40):
            CASES.append((dist, dim, k))


@pytest.mark.parametrize("dist,dim,k", CASES)
def test_grid_equals_bruteforce(dist, dim, k):
    n = 1500 if dim <= 3 else 900
    p = workloads.gen_points(dist, n, dim, 10 * dim + int(k))
    eps = workloads.eps_for_k(dist, n, dim, k)
    a = oracle.bf_pairs(p, eps)
    b = oracle.grid_pairs(p, eps)
    np.testing.assert_array_equal(a, b)
    g = oracle.grid_count(p, eps)
    assert g["count"] == a.shape[0]
    assert g["hash"] == oracle.hash_pairs(a)
    assert g["calcs"] >= g["count"]


def test_grid_equals_bruteforce_sw_shaped():
    p = workloads.sw_shaped(3000, 11)
    for eps in (0.5, 2.0, 7.0):
        np.testing.assert_array_equal(oracle.bf_pairs(p, eps), oracle.grid_pairs(p, eps))


def test_one_cell_and_huge_eps():
    p = workloads.uniform(700, 3, 5)
    for eps in (2.0, 10.0):   # everything in one neighbourhood -> all N(N-1) pairs
        assert oracle.grid_count(p, eps)["count"] == 700 * 699
        assert oracle.bf_count(p, eps)[0] == 700 * 699


def test_rows_match_pairs():
    p = workloads.exponential(2500, 3, 9)
    eps = workloads.eps_for_k("exponential", 2500, 3, 30)
    pairs = oracle.bf_pairs(p, eps)
    rows = np.array([0, 7, 100, 2499, 1234], dtype=np.uint32)
    for fn in (oracle.bf_rows, oracle.grid_rows):
        off, cols = fn(p, eps, rows)
        for r, i in enumerate(rows):
            want = pairs[pairs[:, 0] == i][:, 1]
            np.testing.assert_array_equal(cols[off[r]:off[r + 1]], want)


# ----------------------------------------------------------------- invariants

@pytest.mark.parametrize("dist,dim", [("uniform", 2), ("exponential", 3), ("uniform", 6)])
def test_invariants(dist, dim):
    n = 2000
    p = workloads.gen_points(dist, n, dim, 77)
    e1 = workloads.eps_for_k(dist, n, dim, 10)
    e2 = e1 * 1.3
    r1 = oracle.grid_pairs(p, e1)
    r2 = oracle.grid_pairs(p, e2)
    s1, s2 = _set(r1), _set(r2)
    # irreflexive
    assert not np.any(r1[:, 0] == r1[:, 1])
    # symmetric
    assert s1 == {((k & 0xFFFFFFFF) << 32) | (k >> 32) for k in s1}
    # eps-monotone
    assert s1 <= s2 and len(s2) > len(s1)
    # count with the index == count without it
    assert oracle.grid_count(p, e1)["count"] == oracle.bf_count(p, e1)[0] == len(s1)


def test_neighbourhood_guarantee_of_the_grid():
    # Reading c5: with cells of side w = eps(1+2^-20), every eps-pair lies in cells whose
    # integer coordinates differ by at most 1 in every dimension.
    for dist, dim in (("uniform", 2), ("exponential", 3), ("uniform", 5)):
        n = 1500
        p = workloads.gen_points(dist, n, dim, 5)
        eps = workloads.eps_for_k(dist, n, dim, 20)
        coords, first, ids = oracle.grid_cells(p, eps)
        cell_of = np.empty(n, dtype=np.int64)
        for c in range(coords.shape[0]):
            cell_of[ids[first[c]:first[c + 1]]] = c
        pairs = oracle.bf_pairs(p, eps).astype(np.int64)
        dc = np.abs(coords[cell_of[pairs[:, 0]]] - coords[cell_of[pairs[:, 1]]])
        assert dc.max() <= 1
        # and the cells partition the points
        assert np.array_equal(np.sort(ids), np.arange(n, dtype=np.uint32))


def test_rejects_bad_input():
    with pytest.raises(oracle.OracleError):
        oracle.bf_count(np.array([[0.0, np.nan]]), 1.0)
    with pytest.raises(oracle.OracleError):
        oracle.grid_count(np.zeros((3, 2)), -1.0)
    with pytest.raises(oracle.OracleError):
        oracle.grid_count(np.zeros((3, 9)), 1.0)


def test_workload_generators_are_deterministic():
    a = workloads.get_config("c1").points()
    b = workloads.get_config("c1").points()
    assert a.dtype == np.float64 and a.shape == (10_000, 2)
    np.testing.assert_array_equal(a, b)
    assert math.isclose(workloads.get_config("c1").eps, 0.0319154, rel_tol=1e-5)
    assert math.isclose(workloads.get_config("c3").eps, 9.84745e-4, rel_tol=1e-5)
    assert math.isclose(workloads.get_config("c4").eps, 0.120727, rel_tol=1e-5)


# ----------------------------------------------------------------- the distance-calculation count

def _numpy_cells(p, eps):
    """Cell tuples of reading c5/c6 computed with numpy (independent of oracle.c):
    c_d = floor(fl(fl(x_d - min_d) / w)), w = eps (1 + 2^-20)."""
    w = eps * (1.0 + 2.0 ** -20)
    return np.floor((p - p.min(axis=0)) / w).astype(np.int64)


def _numpy_full_scan_calcs(p, eps):
    """Distance calculations of a full 3^n neighbourhood scan that skips j == i, from the cell
    multiplicities alone: sum_A m_A * (sum_{B in N(A)} m_B) - N, N(A) the 3^n cells around A
    (A included)."""
    import itertools

    cells = _numpy_cells(p, eps)
    uniq, m = np.unique(cells, axis=0, return_counts=True)
    mult = {tuple(c): int(k) for c, k in zip(uniq.tolist(), m.tolist())}
    offs = list(itertools.product((-1, 0, 1), repeat=p.shape[1]))
    tot = 0
    for c, k in mult.items():
        tot += k * sum(mult.get(tuple(a + o for a, o in zip(c, off)), 0) for off in offs)
    return tot - p.shape[0]


@pytest.mark.parametrize("dim,g", [(1, 40), (2, 12), (3, 7), (4, 5), (6, 3)])
def test_grid_calcs_lattice_closed_form(dim, g):
    # unit lattice, eps = 1 - 2^-19: w = eps (1 + 2^-20) < 1, so every point has a cell of its
    # own at its lattice coordinate, and a full 3^n scan evaluates prod_d (neighbours in d) - 1
    # candidates per point: sum over the lattice = prod_d sum_x n_d(x) - g^n = (3g - 2)^n - g^n
    # (n_d = 2 at the two faces, 3 inside).  No pair is within eps (spacing 1).
    p = workloads.lattice(g, dim)
    res = oracle.grid_count(p, 1.0 - 2.0 ** -19)
    assert res["ncells"] == g ** dim
    assert res["count"] == 0
    assert res["calcs"] == (3 * g - 2) ** dim - g ** dim


@pytest.mark.parametrize("dist,dim,n,k", [("uniform", 2, 3000, 30), ("exponential", 3, 3000, 40),
                                          ("uniform", 6, 1500, 20), ("uniform", 1, 2000, 10)])
def test_grid_calcs_equal_cell_multiplicity_count(dist, dim, n, k):
    # the oracle counts its calculations query by query; the same number follows from the cell
    # multiplicities (numpy cells, no oracle code): a dropped / doubled neighbour offset or a
    # counted self-comparison fails here
    p = workloads.gen_points(dist, n, dim, 500 + dim)
    eps = workloads.eps_for_k(dist, n, dim, k)
    res = oracle.grid_count(p, eps, with_hash=False)
    assert res["calcs"] == _numpy_full_scan_calcs(p, eps)
    assert res["ncells"] == np.unique(_numpy_cells(p, eps), axis=0).shape[0]


def test_grid_calcs_sw_shaped_and_duplicates():
    p = workloads.sw_shaped(4000, 21)
    assert oracle.grid_count(p, 1.5, with_hash=False)["calcs"] == _numpy_full_scan_calcs(p, 1.5)
    d = workloads.duplicates(300, 3)
    assert oracle.grid_count(d, 1e-6, with_hash=False)["calcs"] == 300 * 299


# ----------------------------------------------------------------- persistent grid (block rows)

@pytest.mark.parametrize("dist,dim", [("uniform", 2), ("exponential", 3), ("uniform", 6)])
def test_grid_rows_range_equals_rows_and_bruteforce(dist, dim):
    n = 2500 if dim <= 3 else 1200
    p = workloads.gen_points(dist, n, dim, 600 + dim)
    eps = workloads.eps_for_k(dist, n, dim, 25)
    want = oracle.bf_pairs(p, eps)
    keys_want = (want[:, 0].astype(np.uint64) << np.uint64(32)) | want[:, 1].astype(np.uint64)
    with oracle.Grid(p, eps) as g:
        parts = [g.keys_range(lo, min(lo + 333, n)) for lo in range(0, n, 333)]
        off, cols = g.rows_range(17, 29)
    np.testing.assert_array_equal(np.concatenate(parts), keys_want)
    off2, cols2 = oracle.grid_rows(p, eps, np.arange(17, 29, dtype=np.uint32))
    np.testing.assert_array_equal(off, off2)
    np.testing.assert_array_equal(cols, cols2)
