"""Per-kernel summary of one sj_create (the last build in an `ncu --set full` report of
tools/step.py, raw page CSV): duration, DRAM bytes and throughput, issue slots, occupancy,
the busiest pipe.  usage: python tools/build_kernels_summary.py RAW_CSV > summary.txt"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
h, units = rows[0], rows[1]
col = {n: i for i, n in enumerate(h)}


def val(r, name, default=float("nan")):
    i = col.get(name)
    if i is None or i >= len(r):
        return default
    try:
        x = float(r[i].replace(",", ""))
    except ValueError:
        return default
    u = units[i]
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-9, "usecond": 1e-6,
             "msecond": 1e-3, "ns": 1e-9, "us": 1e-6, "ms": 1e-3}.get(u, 1)
    return x * scale


data = rows[2:]
# the last build: from the last bbox_kernel on, join kernels excluded
starts = [k for k, r in enumerate(data) if "bbox_kernel" in r[col["Kernel Name"]]]
data = data[starts[-1]:] if starts else data
pipes = [n for n in h if n.startswith("sm__inst_executed_pipe_") and n.endswith(".avg.pct_of_peak_sustained_active")]
print(f"{'kernel':44s} {'us':>7s} {'DRAM MB':>8s} {'GB/s':>7s} {'issue%':>7s} {'occ%':>6s}  busiest pipe")
tot_t = tot_b = 0.0
for r in data:
    name = r[col["Kernel Name"]]
    if "join_kernel" in name or "compact_" in name:
        continue
    short = name.split("(")[0].replace("void ", "").replace("unnamed>::", "").replace("scan_detail::", "")[:44]
    t = val(r, "gpu__time_duration.sum")
    b = val(r, "dram__bytes_read.sum", 0) + val(r, "dram__bytes_write.sum", 0)
    best = max(pipes, key=lambda p: val(r, p, -1)) if pipes else ""
    print(f"{short:44s} {t * 1e6:7.1f} {b / 1e6:8.1f} {b / t / 1e9 if t else 0:7.0f} "
          f"{val(r, 'sm__inst_issued.avg.pct_of_peak_sustained_active'):7.1f} "
          f"{val(r, 'sm__warps_active.avg.pct_of_peak_sustained_active'):6.1f}  "
          f"{best.replace('sm__inst_executed_pipe_', '').split('.')[0]} {val(r, best):.0f}%")
    tot_t += t
    tot_b += b
print(f"{'sum of build kernels (serialised, cold L2)':44s} {tot_t * 1e6:7.1f} {tot_b / 1e6:8.1f} {tot_b / tot_t / 1e9:7.0f}")
