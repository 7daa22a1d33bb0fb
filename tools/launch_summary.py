"""Aggregate an ncu launch list (gpu__time_duration.sum) by kernel; per-step averages."""
import collections
import csv
import sys


def main(path, steps):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if r and r[0] == "ID"][0]
    h = rows[hi]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    agg = collections.OrderedDict()
    for r in rows[hi + 1:]:
        name = r[ki].split("(")[0].replace("void ", "").replace("sj::<unnamed>::", "").replace("sj::", "")[:int(__import__("os").environ.get("LS_W", "48"))]
        v = float(r[vi].replace(",", ""))
        u = r[ui]
        v = v / 1e3 if u in ("ns", "nsecond") else v * 1e3 if u in ("ms", "msecond") else v
        a = agg.setdefault(name, [0, 0.0])
        a[0] += 1
        a[1] += v
    tot = sum(a[1] for a in agg.values())
    print(f"{path}: total {tot:.1f} us over {sum(a[0] for a in agg.values())} launches")
    for k, (c, v) in sorted(agg.items(), key=lambda x: -x[1][1]):
        print(f"  {v / steps:9.1f} us/step {c / steps:6.1f} launches/step {100 * v / tot:5.1f}%  {k}")


if __name__ == "__main__":
    main(sys.argv[1], float(sys.argv[2]) if len(sys.argv) > 2 else 1.0)
