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


# ---------------------------------------------------------------- exported index (sj_export_index)
# Blob format SJIDX004 (sj_runtime.cu BlobHeader): header fields, then 7 arrays
# (pts, orig, qmap, cellq, runs, cell_lid, chunks) at off[i] with bytes[i].
BLOB_HDR = "<QQiiiiddd8d8Q8QQQQQII7Q7QQ"


def parse_blob(blob):
    """The exported index as numpy arrays: dict(n, dim, key_bits, nc, stride, mins, w, n_cells,
    lookup_hash, orig, qmap (n,2), cellq (M,4), cell_lid (M,), chunks)."""
    import struct

    import numpy as np

    raw = blob.tobytes() if hasattr(blob, "tobytes") else bytes(blob)
    hdr = struct.Struct(BLOB_HDR)
    f = hdr.unpack_from(raw[: hdr.size])
    n, dim = f[1], f[2]
    off, nbytes = f[39:46], f[46:53]

    def arr(i, dt):
        return np.frombuffer(raw[off[i]:off[i] + nbytes[i]], dtype=dt)

    return {
        "n": n, "dim": dim, "key_bits": f[4], "w": f[8], "mins": list(f[9:9 + dim]), "nc": list(f[17:17 + dim]),
        "stride": list(f[25:25 + dim]), "n_cells": f[33], "lookup_hash": f[38],
        "orig": arr(1, np.uint32), "qmap": arr(2, np.uint32).reshape(-1, 2), "cellq": arr(3, np.uint32).reshape(-1, 4),
        "cell_lid": arr(5, np.uint64), "chunks": arr(6, np.uint32),
    }
