"""In-place join time per k (threads per query point): python tools/k_probe.py c3k64 [ks].  Diagnostic."""
import statistics
import sys

import torch

sys.path.insert(0, '.')
import paper_conf_ipps_galletg19_b200 as sj  # noqa: E402
import workloads  # noqa: E402

cfg = workloads.get_config(sys.argv[1])
ks = [int(x) for x in sys.argv[2].split(',')] if len(sys.argv) > 2 else [2, 4, 8, 16, 32]
d = torch.from_numpy(cfg.points()).cuda()
with sj.Handle(d, cfg.eps, k=8) as h:
    n = h.count()
out = torch.empty((n, 2), dtype=torch.int32, device='cuda')
for k in ks:
    ts = []
    for i in range(4):
        with sj.Handle(d, cfg.eps, k=k) as h:
            h.self_join(out, n)
            ts.append(h.stats()['ms_join'])
    print(f'{cfg.name} k={k} join med {statistics.median(ts[1:]):.4f} all', ' '.join('%.3f' % t for t in ts), flush=True)
