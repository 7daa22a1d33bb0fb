import sys, time
import torch
sys.path.insert(0, '.')
import paper_conf_ipps_galletg19_b200 as sj
import workloads
cfg = workloads.get_config('c5')
d = torch.from_numpy(cfg.points()).cuda()
with sj.Handle(d, cfg.eps, k=8) as h:
    n = h.count()
out = torch.empty((n, 2), dtype=torch.int32, device='cuda')
for rep in range(3):
    for opts in ({}, {'blocks_per_sm': 1}, {'blocks_per_sm': 2}, {'blocks_per_sm': 3}, {'grab': 4}, {'k': 16}):
        with sj.Handle(d, cfg.eps, k=opts.get('k', 8)) as h:
            for kk, v in opts.items():
                if kk != 'k': h.set_option(kk, v)
            ts = []
            for i in range(5):
                h.self_join(out, n)
                ts.append(h.stats()['ms_join'])
        print(rep, opts, ' '.join(f'{t:.3f}' for t in ts), flush=True)
