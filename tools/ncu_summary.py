"""Summarise an ncu report (details page) into the handful of numbers DESIGN.md cites."""
import csv
import subprocess
import sys

KEYS = ["Duration", "DRAM Throughput", "Memory Throughput", "L1/TEX Hit Rate", "L2 Hit Rate", "Compute (SM) Throughput",
        "Executed Ipc Active", "Issue Slots Busy", "Achieved Occupancy", "Achieved Active Warps Per SM",
        "Registers Per Thread", "Theoretical Occupancy", "Eligible Warps Per Scheduler", "No Eligible",
        "Warp Cycles Per Issued Instruction", "Avg. Active Threads Per Warp", "Avg. Not Predicated Off Threads Per Warp",
        "Executed Instructions", "Branch Efficiency", "Grid Size", "Block Size", "Static Shared Memory Per Block",
        "Mem Busy", "Max Bandwidth", "L2 Cache Throughput", "L1/TEX Cache Throughput"]


def main(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "details", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    h = rows[0]
    seen = {}
    for r in rows[1:]:
        d = dict(zip(h, r))
        name = d.get("Metric Name", "")
        if name in KEYS and name not in seen:
            seen[name] = f"{d.get('Metric Value', '')} {d.get('Metric Unit', '')}".strip()
    kname = rows[1][h.index("Kernel Name")] if len(rows) > 1 and "Kernel Name" in h else "?"
    print("kernel:", kname[:120])
    for k in KEYS:
        if k in seen:
            print(f"  {k:45s} {seen[k]}")
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rr = list(csv.reader(raw.splitlines()))
    if len(rr) > 2:
        hh, units, vals = rr[0], rr[1], rr[2]
        want = ["dram__bytes_read.sum", "dram__bytes_write.sum", "smsp__thread_inst_executed_per_inst_executed.ratio",
                "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active",
                "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
                "smsp__sass_thread_inst_executed_op_dadd_pred_on.sum",
                "smsp__sass_thread_inst_executed_op_dmul_pred_on.sum",
                "smsp__sass_thread_inst_executed_op_dfma_pred_on.sum", "lts__t_bytes.sum",
                "l1tex__t_bytes.sum", "smsp__warps_issue_stalled_long_scoreboard_per_warp_active.pct"]
        for w in want:
            if w in hh:
                i = hh.index(w)
                print(f"  {w:60s} {vals[i]} {units[i]}")


if __name__ == "__main__":
    for rep in sys.argv[1:]:
        main(rep)
