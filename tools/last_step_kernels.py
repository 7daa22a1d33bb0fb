"""From an ncu --csv metrics log of `tools/step.py CFG 1` (sizing handle + one step), keep the
rows of the last step's build kernels: everything after the sizing join's count launch."""
import csv
import sys

rows = [r for r in csv.reader(l for l in open(sys.argv[1]) if not l.startswith("=="))]
h = rows[0]
ki, ni = h.index("Kernel Name"), h.index("ID")
data = rows[1:]
# launch ids of join kernels: the first is the sizing count, the step's build follows it
joins = sorted({int(r[ni]) for r in data if "join_kernel" in r[ki]})
start = joins[0] if joins else -1
w = csv.writer(sys.stdout)
w.writerow(h)
for r in data:
    if int(r[ni]) > start:
        w.writerow(r)
