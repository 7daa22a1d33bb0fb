"""Experiment: pair joins into a 2x buffer (for the SJ_EXP_2CTR two-counter variant)."""
import sys

import torch

sys.path.insert(0, '.')
import paper_conf_ipps_galletg19_b200 as sj  # noqa: E402
import workloads  # noqa: E402

cfg = workloads.get_config(sys.argv[1])
d = torch.from_numpy(cfg.points()).cuda()
with sj.Handle(d, cfg.eps, k=cfg.k) as h:
    n = h.count()
out = torch.empty((2 * n + 64, 2), dtype=torch.int32, device='cuda')
for rep in range(2):
    with sj.Handle(d, cfg.eps, k=cfg.k) as h:
        pj = []
        for i in range(8):
            h.self_join(out, 2 * n + 64)
            pj.append(h.stats()['ms_join'])
    print(cfg.name, 'pairs2x ', ' '.join(f'{t:.3f}' for t in pj), flush=True)
