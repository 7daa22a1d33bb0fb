"""In-place join time with the output counter (out_blocks=0) vs per-warp output blocks (1), in
one process, alternating: python tools/blk_probe.py c5 [reps].  Diagnostic."""
import statistics
import sys

import torch

sys.path.insert(0, '.')
import paper_conf_ipps_galletg19_b200 as sj  # noqa: E402
import workloads  # noqa: E402

cfg = workloads.get_config(sys.argv[1])
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 6
d = torch.from_numpy(cfg.points()).cuda()
with sj.Handle(d, cfg.eps, k=cfg.k) as h:
    n = h.count()
out = torch.empty((n, 2), dtype=torch.int32, device='cuda')
res = {0: [], 1: []}
for i in range(reps):
    for ob in (0, 1):
        with sj.Handle(d, cfg.eps, k=cfg.k, out_blocks=ob) as h:
            h.self_join(out, n)
            res[ob].append(h.stats()['ms_join'])
for ob, t in res.items():
    print(f'{cfg.name} out_blocks={ob} join med {statistics.median(t):.4f} all', ' '.join('%.3f' % x for x in t), flush=True)
