"""Per-configuration ncu facts for bench.py (profiles/ncu_facts.json): from one `ncu --set full`
capture of the emitting join launch of each configuration (tools/r02_evidence.sh) -- DRAM
traffic per launch, warp execution efficiency, FP64 pipe -- plus the build's DRAM traffic from a
per-kernel metrics pass over one step.  Every entry names its config, source file and date.
usage: r02_facts.py EVIDENCE_DIR PROFILE_TAG"""
import csv
import datetime
import json
import os
import sys

ev, tag = sys.argv[1], sys.argv[2]
path = "profiles/ncu_facts.json"
facts = {}
UNITS = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-9, "usecond": 1e-6, "msecond": 1e-3,
         "ms": 1e-3, "us": 1e-6, "ns": 1e-9, "s": 1.0, "second": 1.0}
when = datetime.datetime.utcnow().strftime("%Y-%m-%dT%H:%MZ")
for f in sorted(os.listdir(ev)):
    if not (f.startswith("ncu_") and f.endswith("_join_raw.csv")):
        continue
    c = f[len("ncu_"):-len("_join_raw.csv")]
    rows = list(csv.reader(open(os.path.join(ev, f))))
    h, u, v = rows[0], rows[1], rows[2]
    get, unit = dict(zip(h, v)), dict(zip(h, u))

    def num(k, scale=True):
        x = float(get[k].replace(",", ""))
        return x * UNITS.get(unit[k], 1) if scale else x
    rd, wr = num("dram__bytes_read.sum"), num("dram__bytes_write.sum")
    facts[c] = {
        "config": c, "traffic_bytes_per_launch": int(rd + wr), "dram_read_bytes": int(rd), "dram_write_bytes": int(wr),
        "wee": round(num("smsp__thread_inst_executed_per_inst_executed.ratio", False) / 32.0, 4),
        "ncu_duration_s": num("gpu__time_duration.sum"),
        "fp64_pipe_pct": num("sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active", False),
        "issue_slots_busy_pct": num("sm__inst_issued.avg.pct_of_peak_sustained_active", False)
        if "sm__inst_issued.avg.pct_of_peak_sustained_active" in get else None,
        "source": f"profiles/{tag}/ncu_{c}_join_summary.txt (ncu --set full, the emitting join launch)",
        "measured": when,
    }
    bf = os.path.join(ev, f"ncu_{c}_build_metrics.csv")
    if os.path.exists(bf):  # per-kernel DRAM bytes of one step's build kernels (everything but the join)
        tot = 0.0
        for r in csv.DictReader(l for l in open(bf) if not l.startswith("==")):
            name, metric = r.get("Kernel Name", ""), r.get("Metric Name", "")
            if "join_kernel" in name or "compact_" in name or metric not in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
                continue
            tot += float(r["Metric Value"].replace(",", "")) * UNITS.get(r.get("Metric Unit", "byte"), 1)
        facts[c]["build_traffic_bytes"] = int(tot)
        facts[c]["build_traffic_source"] = f"profiles/{tag}/ncu_{c}_build_metrics.csv (dram bytes, build kernels of one step)"
json.dump(facts, open(path, "w"), indent=1)
print(json.dumps(facts, indent=1))
