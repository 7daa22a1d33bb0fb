"""CPU tests of the C-ABI library: it loads, exports every declared symbol, its host-only
helpers are right, and without a GPU it fails loudly (no CPU fallback)."""
import itertools

import numpy as np
import pytest

import paper_conf_ipps_galletg19_b200 as sj
from paper_conf_ipps_galletg19_b200 import _lib


def test_exports_every_declared_symbol():
    names = sj.header_functions()
    assert "sj_create" in names and "sj_self_join" in names and "sj_destroy" in names
    for n in names:
        assert hasattr(_lib._lib, n), f"libsj.so does not export {n}"
    assert sj.sj_abi_version() == 3


def test_library_is_sm100a_only():
    import subprocess

    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", sj.lib_path], capture_output=True,
                         text=True).stdout
    assert "sm_100a" in out
    archs = set(a for a in ("sm_80", "sm_86", "sm_89", "sm_90") if a + "." in out)
    assert not archs, archs


@pytest.mark.parametrize("dim", range(1, 9))
def test_forward_offsets_lid_unicomp(dim):
    # P:174 (§III-B): compare with every neighbour cell whose linear id is higher.
    # F = (3^n - 1)/2 (half of the 3^n - 1 neighbours); in 2-D, 4 (Fig. 5).
    offs = sj.sj_forward_offsets(dim).astype(np.int64)
    assert offs.shape == ((3 ** dim - 1) // 2, dim)
    if dim == 2:
        assert offs.shape[0] == 4
    allo = set(itertools.product((-1, 0, 1), repeat=dim)) - {(0,) * dim}
    fw = {tuple(o) for o in offs.tolist()}
    bw = {tuple(-x for x in o) for o in fw}
    assert fw | bw == allo and not (fw & bw)
    # "higher linear id" on a row-major grid with >= 3 cells per dimension, interior origin
    rng = np.random.default_rng(dim)
    nc = rng.integers(3, 9, size=dim)
    stride = np.array([int(np.prod(nc[d + 1:])) for d in range(dim)], dtype=np.int64)
    delta = offs @ stride
    assert np.all(delta > 0)
    # and the first non-zero component is +1
    for o in offs:
        nz = o[o != 0]
        assert nz[0] == 1


def test_forward_offsets_rejects_bad_dim():
    with pytest.raises(sj.SJError):
        sj.sj_forward_offsets(0)
    with pytest.raises(sj.SJError):
        sj.sj_forward_offsets(9)


@pytest.mark.parametrize("nch,world", [(10, 2), (1000, 3), (1001, 8), (5, 4), (64, 2), (1, 1)])
def test_slice_chunks_disjoint_cover(nch, world):
    allc = []
    for r in range(world):
        c = sj.sj_slice_chunks(nch, r, world)
        assert np.all(np.diff(c.astype(np.int64)) > 0)
        # chunk c belongs to rank c mod world
        assert np.all(c % world == r)
        allc.append(c)
    cat = np.concatenate(allc)
    assert np.array_equal(np.sort(cat), np.arange(nch, dtype=np.uint32))
    sizes = [len(c) for c in allc]
    assert max(sizes) - min(sizes) <= 1


def test_batch_chunks_fig1_strided():
    """P:73, Fig. 1: 12 points, nbBatches = 3, each batch 4 points strided across the dataset --
    query q_i (1-based) goes to batch (i - 1) mod 3.  With one point per chunk, the SortByWL-only
    rule (queue = 0) must reproduce exactly that assignment."""
    for l in range(3):
        got = sj.sj_batch_chunks(12, 3, l, queue=0)
        want = [i - 1 for i in range(1, 13) if (i - 1) % 3 == l]
        assert got.tolist() == want and len(got) == 4


@pytest.mark.parametrize("nch,nb", [(12, 3), (1000, 7), (5, 5), (240173, 5), (1, 1), (10, 4)])
@pytest.mark.parametrize("queue", [0, 1])
def test_batch_chunks_partition(nch, nb, queue):
    """Every chunk lands in exactly one batch; WorkQueue batches are contiguous ascending ranges
    of D' (reading c14), SortByWL-only batches are residue classes mod nbBatches."""
    parts = [sj.sj_batch_chunks(nch, nb, l, queue) for l in range(nb)]
    cat = np.concatenate(parts)
    assert np.array_equal(np.sort(cat), np.arange(nch, dtype=np.uint32))
    for l, p in enumerate(parts):
        if queue:
            assert len(p) == 0 or np.array_equal(p, np.arange(p[0], p[0] + len(p), dtype=np.uint32))
            if l and len(p) and len(parts[l - 1]):
                assert p[0] == parts[l - 1][-1] + 1
        else:
            assert np.all(p % nb == l)
    sizes = [len(p) for p in parts]
    assert max(sizes) - min(sizes) <= 1
    with pytest.raises(sj.SJError):
        sj.sj_batch_chunks(nch, nb, nb, queue)


def test_fails_loudly_without_gpu():
    import torch

    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(sj.SJError, match="no CUDA device"):
        sj.sj_create(np.zeros((10, 2)), 0.1)
    with pytest.raises(sj.SJError):
        sj.sj_create_from_index(np.zeros(2048, dtype=np.uint8), 2048)


def test_null_safety():
    sj.sj_destroy(0)
    with pytest.raises(sj.SJError):
        sj.sj_self_join(0, None, 0)
    with pytest.raises(sj.SJError):
        sj.sj_set_slice(0, 0, 1)


def test_argument_validation_before_device():
    with pytest.raises(sj.SJError):
        sj.sj_create(np.zeros((4, 9)), 0.1)       # dim 9
    with pytest.raises(sj.SJError):
        sj.sj_create(np.zeros((4, 2)), -1.0)      # eps <= 0
    with pytest.raises(sj.SJError):
        sj.sj_create(np.zeros((4, 2)), float("nan"))
    with pytest.raises(sj.SJError):
        sj.sj_create(np.zeros((0, 2)), 1.0)       # n = 0
    with pytest.raises(TypeError):
        sj.sj_create(np.zeros((4, 2), dtype=np.float32), 1.0)


def test_oracle_not_imported_by_product():
    import os
    import re

    pkg = os.path.dirname(sj.__file__)
    for root, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".cpp", ".h")):
                txt = open(os.path.join(root, f)).read()
                assert not re.search(r"^\s*(import|from)\s+oracle\b", txt, re.M), f
                assert "oracle.c" not in txt and "liboracle" not in txt, f
