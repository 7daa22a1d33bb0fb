"""The paper's variant study (Tables III-V) re-run on B200 with this library.

    python tools/ablation.py [configs...]            # join times (CUDA events)
    ncu --metrics smsp__thread_inst_executed_per_inst_executed.ratio,gpu__time_duration.sum \
        -k regex:join_kernel --csv python tools/ablation.py --one c3k64 gcg input 1   # WEE of one variant

Variants (Table II): GPUCALCGLOBAL (full 3^n pattern, input order, k=1), UNICOMP,
LID-UNICOMP, k=8, SortByWL (workload-sorted D', static thread assignment), WorkQueue (the
same D' handed out by an atomic counter) and the combination (LID-UNICOMP + WorkQueue + k=8).
"input" order is the paper's unsorted D.
"""
import json
import sys

import torch

sys.path.insert(0, ".")
import paper_conf_ipps_galletg19_b200 as sj  # noqa: E402
import workloads  # noqa: E402

VARIANTS = [  # (label, pattern, order, k, queue): queue 0 = static thread assignment, 1 = WorkQueue
    ("GPUCALCGLOBAL", "gcg", "input", 1, 0),
    ("UNICOMP", "unicomp", "input", 1, 0),
    ("LID-UNICOMP", "lid_unicomp", "input", 1, 0),
    ("GPUCALCGLOBAL k=8", "gcg", "input", 8, 0),
    ("SORTBYWL", "gcg", "workload", 1, 0),
    ("SORTBYWL k=8", "gcg", "workload", 8, 0),
    ("WORKQUEUE", "gcg", "workload", 1, 1),
    ("WORKQUEUE k=8", "gcg", "workload", 8, 1),
    ("WQ + LID-UNICOMP + k=8", "lid_unicomp", "workload", 8, 1),
]


def measure(cfg, d, pattern, order, k, queue, reps=3):
    with sj.Handle(d, cfg.eps, pattern=pattern, order=order, k=k, queue=queue) as h:
        n = h.count()
    out = torch.empty((max(n, 1), 2), dtype=torch.int32, device="cuda")
    ts = []
    for _ in range(reps):
        with sj.Handle(d, cfg.eps, pattern=pattern, order=order, k=k, queue=queue) as h:
            rc, c = h.self_join(out, n)
            assert rc == sj.SJ_OK and c == n
            st = h.stats()
            ts.append(st["ms_join"])
    return min(ts), st, n


def main():
    if len(sys.argv) > 1 and sys.argv[1] == "--one":
        name, pattern, order, k = sys.argv[2], sys.argv[3], sys.argv[4], int(sys.argv[5])
        queue = int(sys.argv[6]) if len(sys.argv) > 6 else 1
        cfg = workloads.get_config(name)
        d = torch.from_numpy(cfg.points()).cuda()
        ms, st, n = measure(cfg, d, pattern, order, k, queue, reps=1)
        print(json.dumps({"config": name, "pattern": pattern, "order": order, "k": k, "queue": queue,
                          "join_ms": ms}))
        return
    names = sys.argv[1:] or ["c2k64", "c3k64", "c4k32", "c5"]
    for name in names:
        cfg = workloads.get_config(name)
        d = torch.from_numpy(cfg.points()).cuda()
        for label, pattern, order, k, queue in VARIANTS:
            ms, st, n = measure(cfg, d, pattern, order, k, queue)
            print(json.dumps({"config": name, "variant": label, "pattern": pattern, "order": order, "k": k,
                              "queue": queue,
                              "join_ms": round(ms, 4), "dist_calcs": st["dist_calcs"], "pairs": n}), flush=True)


if __name__ == "__main__":
    main()
