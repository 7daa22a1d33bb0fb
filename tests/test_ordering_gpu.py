"""Stream ordering and blob validation at the C ABI.  -m gpu.

* Device inputs written asynchronously on the caller's stream (torch's current stream, the
  legacy default one or a side stream) are complete before the library reads them
  (sj_set_stream / the binding's _order_after_torch, include/sj.h "Stream ordering").
* A received index blob is validated field by field (sj_create_from_index): truncated or
  corrupt blobs give SJ_EINVAL instead of out-of-bounds copies.
"""
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
from conftest import BLOB_HDR  # noqa: E402

DEV = "cuda:0"
SLEEP = 200_000_000  # cycles (~0.1 s at 1.9 GHz): the producer is still running when sj_create starts


def _case():
    cfg = workloads.get_config("c3k64").scaled(60_013)
    pts = cfg.points()
    return pts, cfg.eps, oracle.grid_pairs(pts, cfg.eps)


@pytest.mark.parametrize("side_stream", [False, True])
def test_points_written_asynchronously_by_the_caller(side_stream):
    pts, eps, want = _case()
    src = torch.from_numpy(pts).to(DEV)
    torch.cuda.synchronize()
    st = torch.cuda.Stream() if side_stream else torch.cuda.current_stream()
    with torch.cuda.stream(st):
        dst = torch.full_like(src, float("nan"))  # NaN until the producer's copy lands
        torch.cuda._sleep(SLEEP)                  # a slow producer on the caller's stream
        dst.copy_(src * 1.0)
        with sj.Handle(dst, eps, k=8) as h:       # no synchronisation in between
            out = torch.empty((want.shape[0], 2), dtype=torch.int32, device=DEV)
            torch.cuda._sleep(SLEEP)              # the output buffer is still in use upstream
            out.fill_(-1)
            rc, c = h.self_join(out, want.shape[0])
        assert rc == sj.SJ_OK and c == want.shape[0]
        torch.cuda._sleep(SLEEP // 4)
        got = out.cpu().numpy().view(np.uint32)
    np.testing.assert_array_equal(oracle.canonical(got), want)


def test_blob_validation():
    pts, eps, want = _case()
    with sj.Handle(torch.from_numpy(pts).to(DEV), eps) as h:
        nbytes = h.export_index()
        blob = np.empty(nbytes, dtype=np.uint8)
        h.export_index(blob, nbytes)
    hdr = struct.Struct(BLOB_HDR)
    fields = list(hdr.unpack_from(blob.tobytes()))
    with sj.Handle.from_index(blob, nbytes) as ok:  # intact
        assert ok.count() == want.shape[0]

    def corrupt(index, value, size=nbytes):
        f = list(fields)
        f[index] = value
        b = blob.copy()
        hdr.pack_into(b, 0, *f)
        with pytest.raises(sj.SJError) as e:
            sj.Handle.from_index(b, size)
        assert e.value.code == sj.SJ_EINVAL and "bad header" in str(e.value)

    corrupt(0, 0x1234)                      # magic
    corrupt(1, fields[1] * 4)               # n: array sizes no longer match
    corrupt(2, 9)                           # dim
    corrupt(3, 5)                           # pad
    corrupt(33, fields[1] + 1)              # n_cells > n
    corrupt(36, 0)                          # n_chunks
    corrupt(39 + 4, fields[53])             # runs offset past the end
    corrupt(46 + 2, fields[46 + 2] - 8)     # qmap bytes
    corrupt(53, nbytes + 4096)              # total beyond the buffer
    with pytest.raises(sj.SJError):
        sj.Handle.from_index(blob[: nbytes // 2].copy(), nbytes // 2)  # truncated
