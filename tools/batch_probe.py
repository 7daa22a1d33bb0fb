import sys, torch
sys.path.insert(0, '.')
import paper_conf_ipps_galletg19_b200 as sj, workloads
cfg = workloads.get_config(sys.argv[1]); pts = cfg.points(); d = torch.from_numpy(pts).cuda()
h = sj.Handle(d, cfg.eps, k=8, fast_path=0, streams=1, batch_pairs=int(sys.argv[2]))
n = h.count(); out = torch.empty((n, 2), dtype=torch.int32, device='cuda')
for i in range(2):
    rc, c = h.self_join(out, n); print(h.stats()['batches'], h.stats()['ms_join_sum'], file=sys.stderr)
