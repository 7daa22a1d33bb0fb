"""The index the CUDA build writes (a3-a8), checked against definitions computed here with
numpy from the raw points -- not against the kernels' own arithmetic.  -m gpu.

* a3 cell linearisation (readings c5-c7): c_d = floor(fl(fl(x_d - min_d)/w)),
  w = eps (1 + 2^-20), nc_d = max c_d + 1, row-major lid with dimension 0 most significant;
* a5 non-empty cells only: the set of lids and every cell's multiplicity m;
* a6/a7 forward workload ("the number of distance calculations of each non-empty
  cell"): S(A) = sum of m_B over the LID-UNICOMP neighbours B of A (offsets whose first non-zero
  component is +1, Alg. 3), W(A) = floor(m_A/2) + S(A) (reading c9);
* a8 SortByWL: D' is a permutation of the points, every cell's points contiguous,
  cells in non-increasing W, ties by lid (reading c10).
Also the sparse grids whose lookup is the hash table (the paper indexes only the non-empty cells,
P:61), with 32- and 64-bit cell keys, element by element against the oracle.
"""
import itertools

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

import oracle  # noqa: E402
import paper_conf_ipps_galletg19_b200 as sj  # noqa: E402
import workloads  # noqa: E402
from conftest import parse_blob  # noqa: E402
from fullcmp import canonical_blocks_equal  # noqa: E402

DEV = "cuda:0"


def export(h):
    nbytes = h.export_index()
    blob = torch.empty(nbytes, dtype=torch.uint8)
    h.export_index(blob, nbytes)
    return parse_blob(blob.numpy())


def numpy_grid(pts, eps):
    w = eps * (1.0 + 2.0 ** -20)
    cells = np.floor((pts - pts.min(axis=0)) / w).astype(np.int64)
    nc = cells.max(axis=0) + 1
    dim = pts.shape[1]
    stride = [1] * dim
    for d in range(dim - 2, -1, -1):
        stride[d] = stride[d + 1] * int(nc[d + 1])
    lid = np.zeros(pts.shape[0], dtype=np.uint64)
    for d in range(dim):
        lid += cells[:, d].astype(np.uint64) * np.uint64(stride[d])
    return cells, [int(x) for x in nc], stride, lid


def forward_offsets(dim):
    return [o for o in itertools.product((-1, 0, 1), repeat=dim)
            if any(o) and next(x for x in o if x != 0) == 1]


def check_index(pts, eps, B):
    n, dim = pts.shape
    cells, nc, stride, lid = numpy_grid(pts, eps)
    # a3: geometry and linearisation
    assert B["nc"] == nc and B["stride"] == stride
    # a5: the non-empty cells and their multiplicities
    uniq, first, m = np.unique(lid, return_index=True, return_counts=True)
    M = uniq.shape[0]
    assert B["n_cells"] == M
    qm, cq, clid, orig = B["qmap"][:n], B["cellq"][:M], B["cell_lid"][:M], B["orig"][:n]
    pos = np.searchsorted(uniq, clid)
    assert np.all(pos < M) and np.array_equal(uniq[pos], clid), "cell lids"
    assert np.array_equal(np.sort(pos), np.arange(M)), "every non-empty cell once"
    assert np.array_equal(m[pos], cq[:, 1].astype(np.int64)), "cell multiplicities"
    # a8: D' is a permutation of the lid positions; cells contiguous, in queue order 0..M-1
    assert np.array_equal(np.sort(qm[:, 0]), np.arange(n, dtype=np.uint32)), "D' is a permutation"
    qc = qm[:, 1].astype(np.int64)
    assert qc[0] == 0 and np.all(np.diff(qc) >= 0) and np.all(np.diff(qc) <= 1) and qc[-1] == M - 1
    assert np.array_equal(np.bincount(qc, minlength=M), cq[:, 1].astype(np.int64))
    inside = (qm[:, 0] >= cq[qc, 0]) & (qm[:, 0] < cq[qc, 0] + cq[qc, 1])
    assert np.all(inside), "D' position outside its cell's points"
    # every stored point lies in its cell (input id -> numpy lid)
    assert np.array_equal(lid[orig[qm[:, 0]]], clid[qc]), "point in the wrong cell"
    assert np.array_equal(np.sort(orig), np.arange(n, dtype=np.uint32))
    # a6/a7: forward candidates S per cell from the multiplicities
    ucells = cells[first]
    S = np.zeros(M, dtype=np.int64)
    for o in forward_offsets(dim):
        nb = ucells + np.asarray(o, dtype=np.int64)
        ok = np.all((nb >= 0) & (nb < np.asarray(nc)), axis=1)
        nl = np.zeros(M, dtype=np.uint64)
        for d in range(dim):
            nl += np.where(ok, nb[:, d], 0).astype(np.uint64) * np.uint64(stride[d])
        j = np.minimum(np.searchsorted(uniq, nl), M - 1)
        hit = ok & (uniq[j] == nl)
        S += np.where(hit, m[j], 0)
    assert np.array_equal(S[pos], cq[:, 3].astype(np.int64)), "forward workload S"
    # SortByWL: W = floor(m/2) + S non-increasing along the queue, ties by lid
    W = m[pos] // 2 + S[pos]
    assert np.all(W[:-1] >= W[1:]), "D' not in non-increasing workload"
    tie = W[:-1] == W[1:]
    assert np.all(clid[:-1][tie] < clid[1:][tie]), "tie-break by lid"
    return W


IDX_CASES = [("c1", None), ("c2k64", 300_007), ("c3k64", None), ("c4k32", 150_001), ("c5", None)]


@pytest.mark.parametrize("name,n", IDX_CASES)
def test_index_against_numpy_definitions(name, n):
    cfg = workloads.get_config(name)
    if n is not None:
        cfg = cfg.scaled(n)
    pts = cfg.points()
    with sj.Handle(torch.from_numpy(pts).to(DEV), cfg.eps, k=8) as h:
        B = export(h)
        st = h.stats()
    W = check_index(pts, cfg.eps, B)
    # D_alg (a7) from the same multiplicities: sum_A C(m_A, 2) + m_A S(A)
    m = B["cellq"][:, 1].astype(np.int64)
    assert st["dist_calcs"] == int(np.sum(m * (m - 1) // 2 + m * B["cellq"][:, 3].astype(np.int64)))
    assert st["max_cell_load"] == int(W.max())


# ------------------------------------------------------------------ sparse grids: hashed lookup

def sparse_cases():
    out = []
    # 2-D: two dense clusters 1e6 eps apart -> prod nc ~ 1e8 > 64 N: hash table, 27-bit keys
    eps = 0.01
    out.append(("2d-far", workloads.clusters([[0.0, 0.0], [1e6 * eps, 0.0]], 20_000, 0.1, 7), eps, False))
    # 1-D: two clusters 1e8 eps apart (prod nc > 2^27)
    out.append(("1d-far", workloads.clusters([[0.0], [1e5]], 15_000, 0.05, 8), 1e-3, False))
    # 3-D: 3000 tight clusters in the unit cube, eps 5e-4 -> 2000^3 = 8e9 cells: 64-bit keys
    c3 = np.random.default_rng(9).random((3000, 3))
    out.append(("3d-u64", workloads.clusters(c3, 20, 2e-4, 10), 5e-4, True))
    # 6-D: 2000 clusters, eps 0.02 -> ~51^6 = 1.8e10 cells: 64-bit keys
    c6 = np.random.default_rng(11).random((1500, 6))
    out.append(("6d-u64", workloads.clusters(c6, 20, 0.005, 12), 0.02, True))
    return out


@pytest.mark.parametrize("name,pts,eps,wide", sparse_cases(), ids=[c[0] for c in sparse_cases()])
@pytest.mark.parametrize("k", [1, 8])
def test_sparse_grid_hash_lookup(name, pts, eps, wide, k):
    want = oracle.grid_pairs(pts, eps)
    assert want.shape[0] > 5 * pts.shape[0]  # the lookup must find neighbours (hits)
    p = torch.from_numpy(pts).to(DEV)
    with sj.Handle(p, eps, k=k, count_calcs=1) as h:
        st0 = h.stats()
        out = sj.self_join_pairs(h, DEV)
        st = h.stats()
        B = export(h) if k == 8 else None
    assert st0["lookup_hash"] == 1
    assert (st0["key_bits"] > 32) == wide
    np.testing.assert_array_equal(oracle.canonical(out.cpu().numpy().view(np.uint32)), want)
    g = oracle.grid_count(pts, eps, with_hash=False)
    assert st["calcs_measured"] == st["dist_calcs"] == g["calcs"] // 2
    if B is not None:
        check_index(pts, eps, B)


def test_sparse_grid_exact_and_staged():
    name, pts, eps, _ = sparse_cases()[3]
    p = torch.from_numpy(pts).to(DEV)
    with sj.Handle(p, eps, k=8, exact=1) as h:
        out = sj.self_join_pairs(h, DEV)
    canonical_blocks_equal(out, pts, eps, block_pairs=50_000)
    with sj.Handle(p, eps, k=8, fast_path=0, batch_pairs=30_000) as h:
        out = sj.self_join_pairs(h, "cpu")
        assert h.stats()["batches"] > 3
    np.testing.assert_array_equal(oracle.canonical(out.numpy().view(np.uint32)), oracle.grid_pairs(pts, eps))
