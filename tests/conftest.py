import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

GOLDEN = os.path.join(ROOT, "tests", "golden")


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200); run with -m gpu")
    config.addinivalue_line("markers", "slow: full-size configuration (minutes)")


def load_golden(name):
    """Parse a tests/golden fixture: returns (points (N,dim) float64, eps, pairs (M,2) uint32)."""
    import numpy as np

    dim = eps = None
    pts, pairs, mode = [], [], None
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.split("#", 1)[0].strip()
            if not line:
                continue
            tok = line.split()
            if tok[0] == "dim":
                dim = int(tok[1])
            elif tok[0] == "eps":
                eps = float(tok[1])
            elif tok[0] in ("points", "pairs"):
                mode = tok[0]
            elif mode == "points":
                pts.append([float(t) for t in tok])
            elif mode == "pairs":
                pairs.append([int(t) for t in tok])
    p = np.array(pts, dtype=np.float64).reshape(-1, dim)
    q = np.array(pairs, dtype=np.uint32).reshape(-1, 2)
    return p, eps, q
