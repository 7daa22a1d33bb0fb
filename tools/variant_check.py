"""Parity of an experimental libsj variant (SJ_LIB_PATH) vs the oracle on scaled configs (k=8)."""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import oracle  # noqa: E402
import paper_conf_ipps_galletg19_b200 as sj  # noqa: E402
import workloads  # noqa: E402

ok = True
for name, n in [("c5", 80_000), ("c2k64", 60_011), ("c3k64", 50_021), ("c3k256", 40_003), ("c2k16", 70_001)]:
    cfg = workloads.get_config(name).scaled(n)
    pts = cfg.points()
    want = oracle.grid_pairs(pts, cfg.eps)
    d = torch.from_numpy(pts).cuda()
    for opts in ({}, {"exact": 1}, {"fast_path": 0, "batch_pairs": 50_000}, {"queue": 0}):
        with sj.Handle(d, cfg.eps, k=8, count_calcs=1, **opts) as h:
            cnt = h.count()
            got = oracle.canonical(sj.self_join_pairs(h, "cuda").cpu().numpy().view(np.uint32).reshape(-1, 2))
            st = h.stats()
        good = got.shape == want.shape and np.array_equal(got, want) and cnt == want.shape[0] \
            and st["calcs_measured"] == st["dist_calcs"]
        ok &= good
        print(name, opts, "OK" if good else f"FAIL got {got.shape} want {want.shape} cnt {cnt} "
              f"calcs {st['calcs_measured']} vs {st['dist_calcs']}", flush=True)
print("ALL OK" if ok else "FAILURES")
