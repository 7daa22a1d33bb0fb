"""Markdown table of the ablation (tools/gpu_ablation.sh): join times from times.jsonl and the
warp execution efficiency (smsp__thread_inst_executed_per_inst_executed.ratio / 32) from wee.csv.
    python tools/ablation_table.py gpurun_out/ablation > profiles/<round>/ablation/README.md"""
import csv
import json
import os
import sys

d = sys.argv[1]
times = [json.loads(line) for line in open(os.path.join(d, "times.jsonl")) if line.strip()]
wee = {}
wpath = os.path.join(d, "wee.csv")
if os.path.exists(wpath):
    for row in csv.reader(open(wpath)):
        # config, pattern, order, k, queue, then ncu's csv fields ... metric name, unit, value
        if len(row) < 8 or "thread_inst_executed_per_inst_executed" not in ",".join(row):
            continue
        key = (row[0], row[1], row[2], int(row[3]), int(row[4]))
        try:
            wee[key] = float(row[-1].replace(",", "")) / 32.0
        except ValueError:
            pass
print("# Ablation on B200 (the paper's Tables III-V variants, P:266-277)\n")
print("Join kernel only (device-resident output). Time = min of 3 CUDA-event timings (`tools/ablation.py`);")
print("WEE = `smsp__thread_inst_executed_per_inst_executed.ratio / 32` from ncu on the emitting launch")
print("(`tools/gpu_ablation.sh`), the nvprof warp_execution_efficiency equivalent (P:270).  SORTBYWL is")
print("the paper's intermediate step: the workload-sorted D' with static warp -> chunk assignment (P:187-192);")
print("WORKQUEUE hands the same D' out through the atomic counter (P:194-202).\n")
print("| config | variant | distance calcs | join ms | WEE |")
print("|---|---|---|---|---|")
for t in times:
    key = (t["config"], t["pattern"], t["order"], int(t["k"]), int(t["queue"]))
    w = wee.get(key)
    ws = f"{100 * w:.1f} %" if w is not None else "—"
    print(f"| {t['config']} | {t['variant']} | {t['dist_calcs']:.3e} | {t['join_ms']:.3f} | {ws} |")
