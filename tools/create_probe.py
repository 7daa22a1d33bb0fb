import sys, time, torch
sys.path.insert(0, '.')
import paper_conf_ipps_galletg19_b200 as sj, workloads
cfg = workloads.get_config('c5'); pts = cfg.points()
h_pts = torch.from_numpy(pts).pin_memory(); d_pts = h_pts.cuda()
def create(p, tag):
    torch.cuda.synchronize(); t = time.perf_counter(); h = sj.Handle(p, cfg.eps); t1 = time.perf_counter(); h.close(); t2 = time.perf_counter()
    print(f'{tag}: create {1e3*(t1-t):.2f} ms destroy {1e3*(t2-t1):.2f} ms')
for i in range(3): create(h_pts, 'host'); create(d_pts, 'dev ')
h = sj.Handle(h_pts, cfg.eps); n = h.count()
h_out = torch.empty((n, 2), dtype=torch.int32, pin_memory=True)
t = time.perf_counter(); h.self_join(h_out, n); print('staged join', 1e3*(time.perf_counter()-t)); h.close()
for i in range(3): create(h_pts, 'host'); create(d_pts, 'dev ')
d_out = torch.empty((n, 2), dtype=torch.int32, device='cuda')
h = sj.Handle(d_pts, cfg.eps); t = time.perf_counter(); h.self_join(d_out, n); print('fast join', 1e3*(time.perf_counter()-t)); h.close()
for i in range(3): create(h_pts, 'host'); create(d_pts, 'dev ')
