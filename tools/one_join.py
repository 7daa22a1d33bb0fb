"""One count + one emitting join of a config with options given as key=value (ncu driver)."""
import sys
import torch
sys.path.insert(0, '.')
import paper_conf_ipps_galletg19_b200 as sj, workloads
cfg = workloads.get_config(sys.argv[1])
opts = {kv.split('=')[0]: int(kv.split('=')[1]) for kv in sys.argv[2:]}
d = torch.from_numpy(cfg.points()).cuda()
h = sj.Handle(d, cfg.eps, **opts); n = h.count()
out = torch.empty((n, 2), dtype=torch.int32, device='cuda')
rc, c = h.self_join(out, n); print(cfg.name, opts, 'join ms', h.stats()['ms_join'], file=sys.stderr); h.close()
