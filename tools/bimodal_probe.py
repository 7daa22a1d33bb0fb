"""Diagnose the join's slow mode (C5: 0.94 vs 1.7 ms; C5 eps 0.2: 5.4 vs 6.1 ms), printing per
iteration: join ms, a plain write-bandwidth probe on the same output buffer (torch fill), clocks,
power and throttle reasons (NVML).  Phases: A = one handle joined repeatedly; B = build + join +
destroy per iteration (the bench step).   python tools/bimodal_probe.py c5 [iters]"""
import sys
import time

import torch

sys.path.insert(0, '.')
import paper_conf_ipps_galletg19_b200 as sj  # noqa: E402
import workloads  # noqa: E402

try:
    import pynvml
    pynvml.nvmlInit()
    nvh = pynvml.nvmlDeviceGetHandleByIndex(0)
except Exception:  # noqa: BLE001
    nvh = None


def nv():
    if nvh is None:
        return ''
    sm = pynvml.nvmlDeviceGetClockInfo(nvh, pynvml.NVML_CLOCK_SM)
    mem = pynvml.nvmlDeviceGetClockInfo(nvh, pynvml.NVML_CLOCK_MEM)
    pw = pynvml.nvmlDeviceGetPowerUsage(nvh) / 1000
    rs = pynvml.nvmlDeviceGetCurrentClocksEventReasons(nvh)
    tmp = pynvml.nvmlDeviceGetTemperature(nvh, 0)
    return f'sm {sm} mem {mem} {pw:.0f}W {tmp}C reasons 0x{rs:x}'


cfg = workloads.get_config(sys.argv[1])
iters = int(sys.argv[2]) if len(sys.argv) > 2 else 12
d = torch.from_numpy(cfg.points()).cuda()
with sj.Handle(d, cfg.eps, k=cfg.k) as h:
    n = h.count()
out = torch.empty((n, 2), dtype=torch.int32, device='cuda')


def fill_ms():
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    out.fill_(7)
    b.record()
    torch.cuda.synchronize()
    ms = a.elapsed_time(b)
    return ms, out.numel() * 4 / ms / 1e6


print(cfg.name, 'pairs', n, 'out', out.data_ptr() % (1 << 30), flush=True)
with sj.Handle(d, cfg.eps, k=cfg.k) as h:
    for i in range(iters):
        h.self_join(out, n)
        st = h.stats()
        f, gbs = fill_ms()
        print(f'A {i:2d} join {st["ms_join"]:.3f}  fill {f:.3f} ms ({gbs:.0f} GB/s)  {nv()}', flush=True)
for i in range(iters):
    with sj.Handle(d, cfg.eps, k=cfg.k) as h:
        h.self_join(out, n)
        st = h.stats()
    f, gbs = fill_ms()
    print(f'B {i:2d} join {st["ms_join"]:.3f} build {st["ms_build"]:.3f}  fill {f:.3f} ms ({gbs:.0f} GB/s)  {nv()}',
          flush=True)
    time.sleep(0.01)
