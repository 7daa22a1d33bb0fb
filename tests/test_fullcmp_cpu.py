"""The full-size comparison helper (tests/fullcmp.py) on CPU tensors: it accepts the oracle's
own list in any order and rejects a dropped, a duplicated and an altered pair."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

import oracle  # noqa: E402
import workloads  # noqa: E402
from fullcmp import canonical_blocks_equal  # noqa: E402


def _case():
    pts = workloads.exponential(6000, 3, 44)
    eps = workloads.eps_for_k("exponential", 6000, 3, 30)
    pairs = oracle.grid_pairs(pts, eps).astype(np.int32)
    rng = np.random.default_rng(0)
    return pts, eps, pairs[rng.permutation(pairs.shape[0])]


def test_accepts_shuffled_oracle_list_in_blocks():
    pts, eps, pairs = _case()
    t = torch.from_numpy(pairs)
    total, nb = canonical_blocks_equal(t, pts, eps, block_pairs=20_000)
    assert total == pairs.shape[0] and nb > 3


@pytest.mark.parametrize("mutation", ["drop", "duplicate", "alter", "swap"])
def test_rejects_mutations(mutation):
    pts, eps, pairs = _case()
    p = pairs.copy()
    if mutation == "drop":
        p = p[1:]
    elif mutation == "duplicate":
        p = np.concatenate([p, p[:1]])
    elif mutation == "alter":
        p[5, 1] = (p[5, 1] + 1) % pts.shape[0]
    else:  # an unmirrored pair: (i, j) replaced by (j, i) twice
        p[7] = p[7, ::-1]
    with pytest.raises(AssertionError):
        canonical_blocks_equal(torch.from_numpy(np.ascontiguousarray(p)), pts, eps, block_pairs=20_000)
