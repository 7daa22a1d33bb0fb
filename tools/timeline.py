"""GPU timeline of one create+join+destroy step (torch.profiler / CUPTI sees libsj's kernels).

    python tools/timeline.py c5 [steps]

Prints, for the last step, every kernel / memcpy / memset with its start offset from the
step's first GPU activity, its duration and the idle gap before it, then the totals
(busy vs idle).  Diagnostic only; the numbers are not bench values.
"""
import sys
import time

import torch
from torch.profiler import ProfilerActivity, profile

sys.path.insert(0, '.')
import paper_conf_ipps_galletg19_b200 as sj  # noqa: E402
import workloads  # noqa: E402

import os  # noqa: E402

cfg = workloads.get_config(sys.argv[1] if len(sys.argv) > 1 else 'c5')
steps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
# extra Handle options for the timed steps, e.g. TL_KW="out_blocks=1"
kw = {k: int(v) for k, v in (x.split('=') for x in os.environ.get('TL_KW', '').split(',') if x)}
pts = cfg.points()
d = torch.from_numpy(pts).cuda()
h = sj.Handle(d, cfg.eps, k=cfg.k)
n = h.count()
h.close()
out = torch.empty((n, 2), dtype=torch.int32, device='cuda')


def step():
    hh = sj.Handle(d, cfg.eps, k=cfg.k, **kw)
    hh.self_join(out, n)
    st = hh.stats()
    hh.close()
    return st


for _ in range(2):
    step()
torch.cuda.synchronize()
marks = []
with profile(activities=[ProfilerActivity.CUDA, ProfilerActivity.CPU]) as prof:
    for _ in range(steps):
        torch.cuda.synchronize()
        time.sleep(0.02)  # an idle gap that separates the steps on the GPU timeline
        with torch.profiler.record_function('STEP'):
            st = step()
        torch.cuda.synchronize()
evs = [e for e in prof.events() if e.device_type == torch.autograd.DeviceType.CUDA and e.name != 'STEP']
steps_cpu = [e for e in prof.events() if e.name == 'STEP']
last = steps_cpu[-1]
t0c, t1c = last.time_range.start, last.time_range.end
allg = sorted(evs, key=lambda e: e.time_range.start)
# the last step = the GPU activity after the last idle gap of > 10 ms (CPU and GPU clocks may be
# skewed, and sj_create returns before its kernels ran, so the CPU range does not bracket it)
cut = 0
for i in range(1, len(allg)):
    if allg[i].time_range.start - max(e.time_range.end for e in allg[max(0, i - 64):i]) > 10000:
        cut = i
gpu = allg[cut:]
if not gpu:
    print('no gpu events')
    sys.exit(0)
base = gpu[0].time_range.start
prev_end = base
busy = idle = 0.0
print(f'{"start_us":>9} {"dur_us":>8} {"gap_us":>7}  name')
for e in gpu:
    s, t = e.time_range.start, e.time_range.end
    gap = max(0.0, s - prev_end)
    idle += gap
    busy += t - s
    print(f'{s - base:9.1f} {t - s:8.1f} {gap:7.1f}  {e.name[:90]}')
    prev_end = max(prev_end, t)
print(f'span {prev_end - base:.1f} us  busy {busy:.1f} us  idle {idle:.1f} us  (cpu step {t1c - t0c:.1f} us)')
print('stats', {k: st[k] for k in st if k.startswith('ms_')})
