"""Refresh profiles/ncu_facts.json from an evidence directory (tools/gpu_evidence.sh):
per config, the join launch's DRAM traffic, warp execution efficiency, duration and FP64 pipe
utilisation from `ncu --page raw --csv` exports.  usage: update_facts.py EVIDENCE_DIR TAG"""
import csv
import json
import os
import sys

ev, tag = sys.argv[1], sys.argv[2]
path = "profiles/ncu_facts.json"
facts = json.load(open(path)) if os.path.exists(path) else {}
for c in ["c5", "c2k64", "c3k64", "c4k32"]:
    f = os.path.join(ev, f"ncu_{c}_join_raw.csv")
    if not os.path.exists(f):
        continue
    rows = list(csv.reader(open(f)))
    h, u, v = rows[0], rows[1], rows[2]
    get = dict(zip(h, v))
    unit = dict(zip(h, u))

    def num(k, scale_units=True):
        x = float(get[k].replace(",", ""))
        if scale_units:
            x *= {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-9, "usecond": 1e-6,
                  "msecond": 1e-3, "ms": 1e-3, "us": 1e-6, "ns": 1e-9, "s": 1.0}.get(unit[k], 1)
        return x
    rd, wr = num("dram__bytes_read.sum"), num("dram__bytes_write.sum")
    facts[c] = {
        "traffic_bytes_per_launch": int(rd + wr), "dram_read_bytes": int(rd), "dram_write_bytes": int(wr),
        "wee": round(num("smsp__thread_inst_executed_per_inst_executed.ratio", False) / 32.0, 4),
        "ncu_duration_s": num("gpu__time_duration.sum"),
        "fp64_pipe_pct": num("sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active", False),
        "source": f"profiles/{tag}/ncu_{c}_join_summary.txt (ncu --set full, one launch of the emitting join_kernel)",
    }
json.dump(facts, open(path, "w"), indent=1)
print(json.dumps(facts, indent=1))
