import sys, time, torch
sys.path.insert(0, '.')
import paper_conf_ipps_galletg19_b200 as sj, workloads
cfg = workloads.get_config(sys.argv[1]); pts = cfg.points()
# raw D2H bandwidth
x = torch.empty(int(4e9) // 4, dtype=torch.int32, device='cuda'); y = torch.empty_like(x, device='cpu').pin_memory()
for i in range(2):
    torch.cuda.synchronize(); t = time.perf_counter(); y.copy_(x, non_blocking=True); torch.cuda.synchronize()
    print('D2H 4 GB pinned: %.1f GB/s' % (4.0 / (time.perf_counter() - t)))
del x, y
h_pts = torch.from_numpy(pts).pin_memory()
h = sj.Handle(h_pts, cfg.eps, k=8); n = h.count(); h.close()
h_out = torch.empty((n, 2), dtype=torch.int32, pin_memory=True)
for i in range(3):
    torch.cuda.synchronize(); t = time.perf_counter()
    h = sj.Handle(h_pts, cfg.eps, k=8)
    t1 = time.perf_counter()
    rc, c = h.self_join(h_out, n); st = h.stats(); h.close()
    t2 = time.perf_counter()
    print('e2e wall %.1f ms: create %.1f join %.1f | batches %d launches %d est %.2e join_sum %.2f ms' % (
        (t2 - t) * 1e3, (t1 - t) * 1e3, (t2 - t1) * 1e3, st['batches'], st['join_launches'], st['est_pairs'], st['ms_join_sum']))
