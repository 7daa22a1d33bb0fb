"""Join time of one config under option variants (diagnostic): python tools/opt_probe.py c5 grab=1 grab=2 ..."""
import sys

import torch

sys.path.insert(0, '.')
import paper_conf_ipps_galletg19_b200 as sj  # noqa: E402
import workloads  # noqa: E402

cfg = workloads.get_config(sys.argv[1])
d = torch.from_numpy(cfg.points()).cuda()
with sj.Handle(d, cfg.eps, k=cfg.k) as h:
    n = h.count()
out = torch.empty((n, 2), dtype=torch.int32, device='cuda')
for var in sys.argv[2:]:
    opts = dict(kv.split('=') for kv in var.split(',')) if var != 'default' else {}
    opts = {k: int(v) for k, v in opts.items()}
    best, tot, times = 1e9, 0.0, []
    for it in range(6):
        with sj.Handle(d, cfg.eps, **{**{'k': cfg.k}, **opts}) as h:
            h.self_join(out, n)
            st = h.stats()
        times.append(st['ms_join'])
        if it >= 1:
            best = min(best, st['ms_join'])
            tot += st['ms_join']
    print(f'{cfg.name:6s} {var:24s} join best {best:.4f} mean {tot / 5:.4f} ms  fused {st["est_fused"]}  '
          + ' '.join(f'{t:.3f}' for t in times), flush=True)
