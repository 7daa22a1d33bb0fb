import sys, time, torch
sys.path.insert(0, '.')
import paper_conf_ipps_galletg19_b200 as sj, workloads
pts = workloads.uniform(2000, 2, 1); d = torch.from_numpy(pts).cuda()
out = torch.empty((100000, 2), dtype=torch.int32, device='cuda')
for rep in range(3):
    torch.cuda.synchronize(); t = time.perf_counter(); N = 200
    for i in range(N):
        h = sj.Handle(d, 0.01); h.close()
    t1 = time.perf_counter()
    for i in range(N):
        h = sj.Handle(d, 0.01); h.self_join(out, 100000); h.close()
    t2 = time.perf_counter()
    print('create+destroy %.1f us   create+join+destroy %.1f us' % ((t1 - t) / N * 1e6, (t2 - t1) / N * 1e6))
