"""Build time (sj_create, device span) of configs, median of N steps: python tools/build_probe.py c5 c3k64 ..."""
import statistics
import sys

import torch

sys.path.insert(0, '.')
import paper_conf_ipps_galletg19_b200 as sj  # noqa: E402
import workloads  # noqa: E402

for name in sys.argv[1:]:
    cfg = workloads.get_config(name)
    d = torch.from_numpy(cfg.points()).cuda()
    with sj.Handle(d, cfg.eps, k=cfg.k) as h:
        n = h.count()
    out = torch.empty((n, 2), dtype=torch.int32, device='cuda')
    b, j = [], []
    for i in range(12):
        with sj.Handle(d, cfg.eps, k=cfg.k) as h:
            h.self_join(out, n)
            st = h.stats()
        if i >= 2:
            b.append(st['ms_build'])
            j.append(st['ms_join'])
    print(f'{name:7s} build med {statistics.median(b):.4f} min {min(b):.4f}  join med {statistics.median(j):.4f}', flush=True)
