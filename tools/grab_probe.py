import sys, torch
sys.path.insert(0, '.')
import paper_conf_ipps_galletg19_b200 as sj, workloads
cfg = workloads.get_config(sys.argv[1]); d = torch.from_numpy(cfg.points()).cuda()
h = sj.Handle(d, cfg.eps, k=8); n = h.count(); h.close()
out = torch.empty((n, 2), dtype=torch.int32, device='cuda')
for g in [1, 2, 4, 8, 16]:
    ts = []
    for i in range(3):
        h = sj.Handle(d, cfg.eps, k=8, grab=g); h.self_join(out, n); ts.append(h.stats()['ms_join']); h.close()
    print(cfg.name, 'grab', g, 'join ms', ['%.3f' % t for t in ts])
