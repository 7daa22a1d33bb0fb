"""WorkQueue chunks: the build counts and writes the chunk boundaries per queue
CELL (one scan over the M cells); they must equal the per-D'-position rule -- a big cell
(>= 8 points) has a boundary every 32 positions from its first, small cells at every
32-aligned position and where a big cell ended -- recomputed here from the exported index.
Checked on every distribution and on the degenerate inputs, with the pair set vs the oracle.
-m gpu."""
import struct

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


def blob_and_pairs(pts, eps, order="workload"):
    with sj.Handle(torch.from_numpy(np.ascontiguousarray(pts)).to(DEV), eps, k=8, order=order) as h:
        nbytes = h.export_index()
        blob = torch.empty(nbytes, dtype=torch.uint8)
        h.export_index(blob, nbytes)
        pairs = sj.self_join_pairs(h, DEV).cpu().numpy().view(np.uint32).reshape(-1, 2)
    return blob.numpy(), pairs


def cases():
    out = []
    for name, n in [("c1", None), ("c2k64", 60_011), ("c3k64", 50_021), ("c4k32", 20_011), ("c5", 80_000),
                    ("c3k256", 40_003)]:
        cfg = workloads.get_config(name)
        if n is not None:
            cfg = cfg.scaled(n)
        out.append((name, cfg.points(), cfg.eps))
    out.append(("dups-9000", workloads.duplicates(9000, 2), 1e-6))        # one cell > 8192 points
    out.append(("dups-3000", workloads.duplicates(3000, 3), 1e-6))        # one block-sorted cell
    out.append(("one-cell", workloads.uniform(2000, 2, 4), 10.0))
    out.append(("single", np.array([[0.5, 0.5]]), 0.1))
    out.append(("lattice", workloads.lattice(40, 2), 1.0))
    return out


_HDR = struct.Struct("<QQiiiiddd8d8Q8QQQQQII7Q7QQ")


def chunks_by_position(blob):
    """WorkQueue chunk boundaries recomputed from the blob's D' with the per-position rule of
    DESIGN.md §4 (big cell: every 32 positions from its first; small cells: every 32-aligned
    position, and where a big cell ended) -- the definition the per-cell scan must reproduce."""
    raw = blob.tobytes()
    f = _HDR.unpack_from(raw[:_HDR.size])
    n = f[1]
    off, nbytes = f[39:46], f[46:53]
    qmap = np.frombuffer(raw[off[2]:off[2] + nbytes[2]], dtype=np.uint32).reshape(-1, 2)
    cellq = np.frombuffer(raw[off[3]:off[3] + nbytes[3]], dtype=np.uint32).reshape(-1, 4)
    chunks = np.frombuffer(raw[off[6]:off[6] + nbytes[6]], dtype=np.uint32)
    iq = qmap[:n, 1].astype(np.int64)
    m = cellq[iq, 1].astype(np.int64)
    p = np.arange(n, dtype=np.int64)
    beg = np.zeros(n, dtype=np.int64)
    starts = np.r_[True, iq[1:] != iq[:-1]]
    beg[starts] = p[starts]
    beg = np.maximum.accumulate(beg)
    big = m >= 8
    prev_big = np.r_[False, big[:-1]]
    flag = np.where(big, (p - beg) % 32 == 0, (p % 32 == 0) | ((p == beg) & (p > 0) & prev_big))
    want = np.r_[p[flag], n].astype(np.uint32)
    return chunks, want


@pytest.mark.parametrize("name,pts,eps", cases(), ids=[c[0] for c in cases()])
@pytest.mark.parametrize("order", ["workload", "cell"])
def test_chunk_boundaries_per_cell_equal_per_position_rule(name, pts, eps, order):
    blob, pairs = blob_and_pairs(pts, eps, order)
    got, want = chunks_by_position(blob)
    np.testing.assert_array_equal(got, want)
    if order == "workload" and pts.shape[0] <= 80_000 and pairs.shape[0] <= 20_000_000:
        np.testing.assert_array_equal(oracle.canonical(pairs), oracle.grid_pairs(pts, eps))
