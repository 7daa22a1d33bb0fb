"""Which condition selects the join's slow mode?  python tools/bimodal_probe2.py c5 [iters]"""
import sys
import time

import torch

sys.path.insert(0, '.')
import paper_conf_ipps_galletg19_b200 as sj  # noqa: E402
import workloads  # noqa: E402

import threading

try:
    import pynvml
    pynvml.nvmlInit()
    nvh = pynvml.nvmlDeviceGetHandleByIndex(0)
except Exception:  # noqa: BLE001
    nvh = None
samples = []
stop = [False]


def sampler():
    while not stop[0] and nvh is not None:
        samples.append((pynvml.nvmlDeviceGetClockInfo(nvh, pynvml.NVML_CLOCK_SM),
                        pynvml.nvmlDeviceGetClockInfo(nvh, pynvml.NVML_CLOCK_MEM),
                        pynvml.nvmlDeviceGetCurrentClocksEventReasons(nvh)))
        time.sleep(0.0005)


threading.Thread(target=sampler, daemon=True).start()
cfg = workloads.get_config(sys.argv[1])
iters = int(sys.argv[2]) if len(sys.argv) > 2 else 12
d = torch.from_numpy(cfg.points()).cuda()
with sj.Handle(d, cfg.eps, k=cfg.k) as h:
    n = h.count()
out = torch.empty((n, 2), dtype=torch.int32, device='cuda')
out2 = torch.empty((n, 2), dtype=torch.int32, device='cuda')
flush = torch.empty(256 << 20, dtype=torch.uint8, device='cuda')
flush.fill_(1)
out.fill_(0)
out2.fill_(0)
torch.cuda.synchronize()


def run(name, between=None, alt=False, fresh=False):
    ts = []
    samples.clear()
    with sj.Handle(d, cfg.eps, k=cfg.k) as h:
        for i in range(iters):
            o = out2 if (alt and i % 2) else out
            if fresh:
                o = torch.empty((n, 2), dtype=torch.int32, device='cuda')
            h.self_join(o, n)
            ts.append(h.stats()['ms_join'])
            if between:
                between()
            del o
    sm = [x[0] for x in samples] or [0]
    rs = 0
    for x in samples:
        rs |= x[2]
    print(f'{cfg.name} {name:14s} ' + ' '.join(f'{t:.3f}' for t in ts) +
          f'  | sm min {min(sm)} max {max(sm)} n {len(sm)} reasons 0x{rs:x}', flush=True)


run('back2back')
run('sleep0.2', lambda: time.sleep(0.2))
run('flush256M', lambda: (flush.fill_(3), torch.cuda.synchronize()))
run('alt-buffers', alt=True)
run('back2back')
run('sync-only', lambda: torch.cuda.synchronize())
stop[0] = True
