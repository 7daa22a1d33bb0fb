"""Join time along the WorkQueue: the in-place join of consecutive sub-ranges of D' chunks
(SJ_DEBUG_VRANGE), with the pairs each emits and the achieved write bandwidth.  Diagnostic.
    SJ_DEBUG_VRANGE is set per sub-range by re-exec; usage: python tools/vrange_profile.py c5 [parts]"""
import os
import subprocess
import sys

import torch

sys.path.insert(0, '.')
import paper_conf_ipps_galletg19_b200 as sj  # noqa: E402
import workloads  # noqa: E402

cfg = workloads.get_config(sys.argv[1])
parts = int(sys.argv[2]) if len(sys.argv) > 2 else 10
if 'VR_CHILD' not in os.environ:
    d = torch.from_numpy(cfg.points()).cuda()
    h = sj.Handle(d, cfg.eps, k=cfg.k)
    tot = h.count()
    V = h.stats()['n_chunks']
    h.close()
    print(f'{cfg.name}: {V} chunks, {tot} pairs')
    cuts = [V * i // parts for i in range(parts + 1)]
    for a, b in zip(cuts, cuts[1:]):
        env = dict(os.environ, VR_CHILD='1', SJ_DEBUG_VRANGE=f'{a},{b}')
        out = subprocess.run([sys.executable, __file__, sys.argv[1]], env=env, capture_output=True, text=True)
        print(f'[{a:7d},{b:7d}) ' + out.stdout.strip() + out.stderr.strip()[-300:])
else:
    d = torch.from_numpy(cfg.points()).cuda()
    h = sj.Handle(d, cfg.eps, k=cfg.k)
    n = h.count()
    out = torch.empty((n, 2), dtype=torch.int32, device='cuda')
    best = 1e9
    for _ in range(3):
        h.self_join(out, n)
        st = h.stats()
        best = min(best, st['ms_join'])
    print(f'pairs {st["pairs"]:11d}  join {best:.4f} ms  {st["pairs"] * 8 / best / 1e6:8.1f} GB/s')
    h.close()
