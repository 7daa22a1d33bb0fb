"""Small driver for compute-sanitizer (memcheck / racecheck / synccheck / initcheck): every join
path on C1 and a 1e5-point C3 -- in-place fast path (fused estimator), staged batches with
forced overflow retries, exact two-pass sizing, SJ_MORE continuation into a host buffer,
count-only, device CSR, the slab-partition calls -- each checked against the oracle so a
sanitizer run is also a parity run.  usage: python tools/sanitize_driver.py [small]"""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import oracle  # noqa: E402
import paper_conf_ipps_galletg19_b200 as sj  # noqa: E402
import workloads  # noqa: E402
from paper_conf_ipps_galletg19_b200 import dist as sjdist  # noqa: E402

small = len(sys.argv) > 1 and sys.argv[1] == "small"
cases = [workloads.get_config("c1")]
if not small:
    cases.append(workloads.get_config("c3k64").scaled(100_003))


def canon(t):
    return oracle.canonical(t.cpu().numpy().view(np.uint32) if hasattr(t, "cpu") else t)


for cfg in cases:
    pts = cfg.points()
    want = oracle.grid_pairs(pts, cfg.eps)
    d = torch.from_numpy(pts).cuda()
    # 1. in-place fast path (device-sized lazy launch with the fused estimator)
    out = torch.empty((want.shape[0], 2), dtype=torch.int32, device="cuda")
    with sj.Handle(d, cfg.eps, k=8) as h:
        rc, c = h.self_join(out, want.shape[0])
    assert rc == sj.SJ_OK and np.array_equal(canon(out[:c]), want), "in place"
    # 2. staged batches, tiny b_s and a tiny estimator sample: overflow retries
    with sj.Handle(d, cfg.eps, k=8, fast_path=0, batch_pairs=7_000, sample_ppm=1) as h:
        got = sj.self_join_pairs(h, "cuda")
        print(cfg.name, "staged: batches", h.stats()["batches"], "retries", h.stats()["retries"], flush=True)
    assert np.array_equal(canon(got), want), "staged"
    # 3. exact two-pass sizing, staged and in place
    for fp in (0, 1):
        with sj.Handle(d, cfg.eps, k=8, exact=1, fast_path=fp, batch_pairs=20_000) as h:
            got = sj.self_join_pairs(h, "cuda")
        assert np.array_equal(canon(got), want), "exact"
    # 4. SJ_MORE continuation into a pageable host buffer
    with sj.Handle(d, cfg.eps, k=8, batch_pairs=9_000) as h:
        buf = np.empty((3_001, 2), dtype=np.uint32)
        parts, rc = [], sj.SJ_MORE
        while rc == sj.SJ_MORE:
            rc, c = h.self_join(buf, 3_001)
            parts.append(buf[:c].copy())
    assert np.array_equal(canon(np.concatenate(parts)), want), "SJ_MORE"
    # 5. count-only, an undersized device buffer (in-place overflow -> staged)
    with sj.Handle(d, cfg.eps, k=4) as h:
        assert h.count() == want.shape[0]
        small_out = torch.empty((want.shape[0] // 2, 2), dtype=torch.int32, device="cuda")
        parts, rc = [], sj.SJ_MORE
        while rc == sj.SJ_MORE:
            rc, c = h.self_join(small_out, small_out.shape[0])
            parts.append(small_out[:c].cpu().numpy().view(np.uint32).copy())
    assert np.array_equal(canon(np.concatenate(parts)), want), "overflow"
    # 5b. blocked in-place output (per-warp output blocks + compaction), exact and larger buffers
    for slack in (0, 999):
        ob = torch.full((want.shape[0] + slack, 2), -1, dtype=torch.int32, device="cuda")
        with sj.Handle(d, cfg.eps, k=8, out_blocks=1) as h:
            rc, c = h.self_join(ob, want.shape[0] + slack)
        assert rc == sj.SJ_OK and np.array_equal(canon(ob[:c]), want), "blocked"
    # 5c. zero-copy index view
    with sj.Handle(d, cfg.eps, k=8) as h:
        nb = h.export_index()
        blob = torch.empty(nb, dtype=torch.uint8, device="cuda")
        h.export_index(blob, nb)
    with sj.Handle.from_index(blob, nb, view=True) as h:
        assert np.array_equal(canon(sj.self_join_pairs(h, "cuda")), want), "view"
    # 6. device CSR on the GCG pattern
    with sj.Handle(d, cfg.eps, pattern="gcg", k=8) as h:
        off, nb = h.neighbor_csr()
    assert int(off[-1]) == want.shape[0]
    # 7. SortByWL-only static assignment
    with sj.Handle(d, cfg.eps, k=8, queue=0) as h:
        got = sj.self_join_pairs(h, "cuda")
    assert np.array_equal(canon(got), want), "queue=0"
    # 8. slab partition arithmetic
    lib = sjdist.LibRouter()
    mn, mx = lib.bounds(d)
    ncol = lib.columns(mn[0], mx[0], cfg.eps)
    hist = lib.histogram(d, mn[0], cfg.eps, ncol)
    lib.pack(d, None, mn[0], cfg.eps, hist, 3)
    torch.cuda.synchronize()
    print(cfg.name, "ok", want.shape[0], "pairs", flush=True)
print("sanitize driver done")
