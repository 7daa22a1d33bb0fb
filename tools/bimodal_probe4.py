"""Count-only joins (no output, no emission atomics) vs pair joins, repeated: does the slow mode
need the output's atomics?   python tools/bimodal_probe4.py c5e02 [iters]"""
import sys

import torch

sys.path.insert(0, '.')
import paper_conf_ipps_galletg19_b200 as sj  # noqa: E402
import workloads  # noqa: E402

cfg = workloads.get_config(sys.argv[1])
iters = int(sys.argv[2]) if len(sys.argv) > 2 else 8
d = torch.from_numpy(cfg.points()).cuda()
with sj.Handle(d, cfg.eps, k=cfg.k) as h:
    n = h.count()
out = torch.empty((n, 2), dtype=torch.int32, device='cuda')
for rep in range(2):
    with sj.Handle(d, cfg.eps, k=cfg.k) as h:
        cnt = []
        for i in range(iters):
            h.count()
            cnt.append(h.stats()['ms_join'])
        pj = []
        for i in range(iters):
            h.self_join(out, n)
            pj.append(h.stats()['ms_join'])
    print(cfg.name, 'count ', ' '.join(f'{t:.3f}' for t in cnt), flush=True)
    print(cfg.name, 'pairs ', ' '.join(f'{t:.3f}' for t in pj), flush=True)
