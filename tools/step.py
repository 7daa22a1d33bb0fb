"""Run a few create+join+destroy steps of a config (debug / ncu driver)."""
import sys
import time

import torch

sys.path.insert(0, '.')
import paper_conf_ipps_galletg19_b200 as sj  # noqa: E402
import workloads  # noqa: E402

cfg = workloads.get_config(sys.argv[1])
steps = int(sys.argv[2]) if len(sys.argv) > 2 else 4
k = int(sys.argv[3]) if len(sys.argv) > 3 else cfg.k
pts = cfg.points()
d = torch.from_numpy(pts).cuda()
h = sj.Handle(d, cfg.eps, k=k)
n = h.count()
h.close()
out = torch.empty((n, 2), dtype=torch.int32, device='cuda')
for i in range(steps):
    torch.cuda.synchronize()
    t = time.perf_counter()
    h = sj.Handle(d, cfg.eps, k=k)
    rc, c = h.self_join(out, n)
    st = h.stats()
    h.close()
    torch.cuda.synchronize()
    print(cfg.name, 'k', k, 'step wall ms %.3f' % ((time.perf_counter() - t) * 1e3), 'join %.3f' % st['ms_join'],
          'build %.3f' % st['ms_build'], 'est %.3f' % st['ms_estimate'], 'fast', st['fast_path'], file=sys.stderr)
