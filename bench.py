#!/usr/bin/env python
"""bench.py -- B200 eps-grid self-join throughput (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c5] [--k 8]
    python bench.py --impl reference ...      # the CPU oracle on the host cores

A step is one pass of the whole hot path (DESIGN.md §1 a1..a12) over the synthetic
workload with the points already resident in HBM: sj_create (bbox, cell ids, radix
sort, compaction, forward neighbours, workload, SortByWL) + sj_self_join (estimator,
join into an HBM result buffer) + sj_destroy; for N > 1 also the NCCL broadcast of the
index blob and the all-reduce of counts.  value = algorithmic distance calculations
(D_alg, LID-UNICOMP) of the whole job / time.  e2e repeats the step through the same
C ABI from pinned HOST buffers (H2D of the points and D2H of every pair inside the
timed region).  One JSON line is printed by rank 0.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import workloads  # noqa: E402

PEAKS_FILE = os.path.join(ROOT, "MEASURED_PEAKS.json")
FALLBACK_HBM_GBS = 6650.0


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="c5")
    ap.add_argument("--k", type=int, default=None)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--batched-steps", type=int, default=5)
    ap.add_argument("--mp", default="replicated", choices=["replicated", "broadcast"],
                    help="N > 1: every rank builds the index (replicated input), or rank 0 builds and "
                         "NCCL-broadcasts it (zero-copy views on the other ranks)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--ref-stride", type=int, default=0, help="oracle sample: every s-th query (0 = auto)")
    ap.add_argument("--json-out", default=None)
    return ap.parse_args()


# ----------------------------------------------------------------------------- clocks

class ClockSampler:
    """nvidia-smi clocks/throttle sampling during the timed region (B200_PROFILING.md)."""

    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self.proc = None
        self.thread = None

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-lms", "20"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except OSError:
            self.proc = None
            return
        self.thread = threading.Thread(target=self._read, daemon=True)
        self.thread.start()

    def _read(self):
        for line in self.proc.stdout:
            parts = [p.strip() for p in line.split(",")]
            if len(parts) >= 8:
                self.rows.append(parts)

    def stop(self):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()
        if self.thread:
            self.thread.join(timeout=5)

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"], "samples": 0}

        def num(x):
            try:
                return float(x)
            except ValueError:
                return None

        sm = [num(r[0]) for r in self.rows if num(r[0]) is not None]
        smax = [num(r[1]) for r in self.rows if num(r[1]) is not None]
        pw = [num(r[2]) for r in self.rows]
        loaded = [s for s, p in zip(sm, pw) if p is not None and p > 250.0] or sm
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4) if r[4 + i].lower() == "active"})
        return {"sm_mhz": statistics.median(loaded) if loaded else None, "sm_max_mhz": max(smax) if smax else None,
                "reasons": reasons, "samples": len(self.rows), "samples_under_load": len(loaded),
                "power_w_max": max([p for p in pw if p is not None], default=None)}


# ----------------------------------------------------------------------------- helpers

def load_peaks():
    try:
        with open(PEAKS_FILE) as f:
            pk = json.load(f)
        return float(pk["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except (OSError, KeyError, ValueError):
        return FALLBACK_HBM_GBS, "fallback (B200_PROFILING.md)"


def load_profile_facts(cfg_name: str):
    """ncu facts of THIS configuration (DRAM traffic per launch, warp execution efficiency),
    committed under profiles/ by tools/r02_facts.py from an `ncu --set full` capture of the same
    launch in a separate process (bench numbers are never taken under a profiler).  Each entry
    names its source file and capture date; a configuration without its own capture gets none
    (no other configuration's numbers are reused)."""
    p = os.path.join(ROOT, "profiles", "ncu_facts.json")
    try:
        with open(p) as f:
            e = json.load(f).get(cfg_name, {})
    except (OSError, ValueError):
        return {}
    return e if e.get("config") == cfg_name else {}


def build_algorithmic_bytes(st: dict, dim: int, pad: int) -> int:
    """Compulsory HBM bytes of the build (a2-a8): the raw points read once and the
    index written once -- points in cell order (8*pad), input ids (4) and D' (8) per point, the
    cell record (16) and lid (8) per cell, 8 B per forward run slot, 4 B per WorkQueue chunk.
    The sort passes and temporaries are the build's own overhead, not counted."""
    n, m, e, c = st["n"], st["n_cells"], st["fwd_runs"], st["n_chunks"]
    return n * 8 * dim + n * (8 * pad + 12) + m * 24 + 8 * e + 4 * (c + 1)


def pcie_rates(dev, nbytes: int = 1 << 30):
    """Measured pinned host<->device copy rates (bytes/s), best of 3 (the e2e denominator)."""
    import torch

    h = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
    d = torch.empty(nbytes, dtype=torch.uint8, device=dev)
    out = {}
    for name, dst, src in (("h2d", d, h), ("d2h", h, d)):
        best = float("inf")
        for _ in range(3):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            a.record()
            dst.copy_(src, non_blocking=True)
            b.record()
            torch.cuda.synchronize()
            best = min(best, a.elapsed_time(b) * 1e-3)
        out[name] = nbytes / best
    del h, d
    return out


def o1_c1_timing():
    """O1 brute force (two nested loops over all ordered pairs) on C1, timed on the
    host cores: the SURVEY §8(d) brute-force reference point."""
    import oracle

    cfg = workloads.get_config("c1")
    pts = cfg.points()
    t0 = time.perf_counter()
    cnt, _ = oracle.bf_count(pts, cfg.eps)
    dt = time.perf_counter() - t0
    n = pts.shape[0]
    return {"config": "c1", "pairs": cnt, "distance_calcs": n * (n - 1), "seconds": dt,
            "calcs_per_s": n * (n - 1) / dt, "cores": oracle.num_threads()}


def algorithmic_bytes(st: dict, pad: int) -> int:
    """Compulsory HBM bytes of one join launch: every ordered pair written once
    (8 B) plus the index read once: points (pad*8 B), orig id (4 B) and the D' entry (8 B) per
    point, 16 B per cell record, 8 B per forward run."""
    n, m, e = st["n"], st["n_cells"], st["fwd_runs"]
    return 8 * st["pairs"] + n * (8 * pad + 12) + 16 * m + 8 * e


def oracle_baseline(pts, eps, d_alg: int, stride: int, budget_s: float = 20.0, threads: int = 0):
    """The CPU oracle (O2 grid, as it stands) on a strided sample of the queries; threads > 0
    limits its OpenMP threads for this call (the 1-core run)."""
    import oracle

    if threads:
        full = oracle.num_threads()
        oracle.set_threads(threads)
        try:
            return oracle_baseline(pts, eps, d_alg, stride, budget_s, 0)
        finally:
            oracle.set_threads(full)
    n = pts.shape[0]
    if stride <= 0:
        # calibrate on a tiny sample so the measured call lands near budget_s
        s0 = max(n // 2000, 1)
        t0 = time.perf_counter()
        oracle.grid_rows(pts, eps, np.arange(0, n, s0, dtype=np.uint32))
        dt = time.perf_counter() - t0
        per_row = dt / len(range(0, n, s0))
        stride = max(1, int(np.ceil(n * per_row / budget_s)))
    for _attempt in range(3):
        rows = np.arange(0, n, stride, dtype=np.uint32)
        t0 = time.perf_counter()
        off, _ = oracle.grid_rows(pts, eps, rows)
        dt = time.perf_counter() - t0
        # the calibration call is dominated by the grid build: widen the sample until it is
        # a budget's worth of work (or every query)
        if dt >= 0.5 * budget_s or stride == 1:
            break
        stride = max(1, int(stride * dt / budget_s))
    frac = rows.shape[0] / n
    return {
        "value": d_alg * frac / dt, "unit": "calcs/s", "cores": oracle.num_threads(), "kind": "oracle",
        "sample": f"O2 grid oracle (hash grid build + full 3^n scan + sorted rows) for every {stride}-th query "
                  f"({rows.shape[0]} of {n} queries, {int(off[-1])} pairs), throughput scaled by the sample "
                  f"fraction {frac:.4f}; {dt:.2f} s",
        "seconds": dt, "stride": stride,
    }


# ----------------------------------------------------------------------------- reference arm

def run_reference(args, rank: int, world: int):
    """--impl reference: the oracle on the box's host cores (rank 0 only)."""
    if rank != 0:
        return
    import oracle

    cfg = workloads.get_config(args.config)
    pts = cfg.points()
    g = oracle.grid_count(pts, cfg.eps, with_hash=False)  # untimed: D_alg of the workload = calcs_GCG / 2
    d_alg = g["calcs"] // 2
    vals, secs = [], []
    base = None
    for i in range(args.warmup + args.steps):
        budget = max(2.0, 150.0 / (args.warmup + args.steps))
        r = oracle_baseline(pts, cfg.eps, d_alg, args.ref_stride if base is None else base["stride"], budget)
        if base is None:
            base = {"stride": r["stride"]}
        if i >= args.warmup:
            vals.append(r["value"])
            secs.append(r["seconds"])
    v = statistics.median(vals)
    line = {
        "impl": "reference", "metric": "distance calcs/s", "value": v, "unit": "calcs/s", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * statistics.median(secs),
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic (seeded, SURVEY.md §8.0)",
        "config": {"workload": f"{cfg.name}: {cfg.note}", "n": cfg.n, "dim": cfg.dim, "eps": cfg.eps,
                   "dist_calcs": d_alg, "pairs": g["count"]},
        "cpu_baseline": {"value": v, "unit": "calcs/s", "cores": oracle.num_threads(), "kind": "oracle",
                         "sample": r["sample"]},
        "e2e": {"value": v, "unit": "calcs/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "gpu_launches": 0,
    }
    emit(line, args)


def emit(line: dict, args):
    s = json.dumps(line)
    print(s, flush=True)
    if args.json_out:
        with open(args.json_out, "a") as f:
            f.write(s + "\n")


# ----------------------------------------------------------------------------- our arm

def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        return run_reference(args, rank, world)

    import torch
    import torch.distributed as dist

    import paper_conf_ipps_galletg19_b200 as sj
    from paper_conf_ipps_galletg19_b200 import dist as sjdist

    assert torch.cuda.is_available(), "bench.py needs a CUDA device"
    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    group = None

    cfg = workloads.get_config(args.config)
    k = args.k or cfg.k
    pts = cfg.points()
    d_pts = torch.from_numpy(pts).to(dev)
    pad = 1 if cfg.dim == 1 else (cfg.dim + 1) & ~1
    flush_buf = torch.empty(256 << 20, dtype=torch.uint8, device=dev)  # > 126 MB L2

    def build():
        if world == 1:
            h = sj.Handle(d_pts, cfg.eps, k=k)
            return h
        if args.mp == "replicated":  # every rank builds from its own copy
            h = sj.Handle(d_pts, cfg.eps, k=k)
        else:  # rank 0 builds; NCCL broadcast of the index blob; zero-copy views elsewhere
            h = sj.Handle(d_pts, cfg.eps, k=k) if rank == 0 else None
            h, _ = sjdist.replicate_index(h, 0, group, dev)
            if rank != 0:
                h.set_option("k", k)
        h.set_slice(rank, world)
        return h

    # sizing (untimed): this rank's slice count
    h = build()
    local_pairs = h.count()
    st0 = h.stats()
    h.close()
    cap = max(local_pairs, 1)
    out = torch.empty((cap, 2), dtype=torch.int32, device=dev)

    def step(out_buf, cap_):
        h = build()
        rc, c = h.self_join(out_buf, cap_)
        st = h.stats()
        h.close()
        if world > 1:
            tot = sjdist.allreduce_counts([c], group, dev)[0]
        else:
            tot = c
        return rc, c, tot, st

    stream = torch.cuda.current_stream()
    sampler = ClockSampler(local_rank)
    sampler.start()
    for _ in range(args.warmup):
        step(out, cap)
    torch.cuda.synchronize()

    # timed region: K steps, L2 flushed before each (excluded from the step events)
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    join_ms, build_ms, est_ms, tot_pairs = [], [], [], None
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    l0 = sj.sj_kernel_launches()
    for i in range(args.steps):
        # the flush is queued on this stream before the step's start event, and every libsj call
        # waits for this stream first (include/sj.h, stream ordering): none of the step's GPU
        # work can start before the flush ended or before the start event
        flush_buf.fill_(i & 0xFF)
        evs[i][0].record(stream)
        rc, c, tot, st = step(out, cap)
        evs[i][1].record(stream)
        assert rc == sj.SJ_OK and c == local_pairs, (rc, c, local_pairs)
        join_ms.append(st["ms_join"])
        build_ms.append(st["ms_build"])
        est_ms.append(st["ms_estimate"])
        tot_pairs = tot
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    launches = sj.sj_kernel_launches() - l0
    step_ms = [a.elapsed_time(b) for a, b in evs]
    total_ms = sum(step_ms)
    step_sorted = sorted(step_ms)
    if world > 1:
        total_ms = sjdist.allreduce_counts([int(total_ms * 1e6)], group, dev, op=dist.ReduceOp.MAX)[0] / 1e6
    sampler.stop()
    clocks = sampler.summary()

    d_alg = st0["dist_calcs"]
    value = d_alg * args.steps / (total_ms * 1e-3)

    # roofline of the dominant kernel (the join): algorithmic bytes / mean launch duration
    hbm_peak, peak_src = load_peaks()
    fp64_peak, _ = sj.sj_measure_fp64()
    st_last = dict(st)
    st_last["pairs"] = local_pairs
    abytes = algorithmic_bytes(st_last, pad)
    mean_join_ms = statistics.mean(join_ms)
    achieved = abytes / (mean_join_ms * 1e-3) / 1e9
    fp64_instr = 3 * cfg.dim * (d_alg / world)
    t_hbm = abytes / (hbm_peak * 1e9)
    t_fp64 = fp64_instr / fp64_peak
    facts = load_profile_facts(cfg.name)
    if t_hbm >= t_fp64:
        roof = {"bound": "hbm", "achieved": achieved, "peak": hbm_peak, "unit": "GB/s", "frac": achieved / hbm_peak,
                "traffic": facts.get("traffic_bytes_per_launch"), "peak_source": peak_src,
                "algorithmic_bytes_per_launch": abytes, "kernel": "join_kernel", "kernel_ms": mean_join_ms}
    else:
        ach = fp64_instr / (mean_join_ms * 1e-3) / 1e12
        roof = {"bound": "fp64", "achieved": ach, "peak": fp64_peak / 1e12, "unit": "Tinstr/s",
                "frac": ach * 1e12 / fp64_peak, "traffic": facts.get("traffic_bytes_per_launch"),
                "peak_source": "measured on this GPU (sj_measure_fp64: DMUL+DADD chains, all SMs)",
                "algorithmic_fp64_instr_per_launch": fp64_instr, "kernel": "join_kernel", "kernel_ms": mean_join_ms}
    roof["fp64_frac"] = (fp64_instr / (mean_join_ms * 1e-3)) / fp64_peak
    roof["hbm_frac"] = achieved / hbm_peak
    roof["fp64_peak_instr_per_s"] = fp64_peak
    if facts:
        roof["traffic_source"] = f"{facts.get('source')} ({facts.get('measured')})"
    # the build (a2-a8) and the whole step against the HBM roofline, compulsory bytes only
    bbytes = build_algorithmic_bytes(st0, cfg.dim, pad)
    mean_build_ms = statistics.mean(build_ms)
    build_roof = {"bound": "hbm", "algorithmic_bytes": bbytes, "ms": mean_build_ms,
                  "achieved": bbytes / (mean_build_ms * 1e-3) / 1e9, "peak": hbm_peak, "unit": "GB/s"}
    build_roof["frac"] = build_roof["achieved"] / hbm_peak
    if facts.get("build_traffic_bytes"):
        build_roof["traffic"] = facts["build_traffic_bytes"]
    step_bytes = abytes + bbytes
    step_roof = {"bound": "hbm", "algorithmic_bytes": step_bytes, "ms": total_ms / args.steps,
                 "achieved": step_bytes / (total_ms / args.steps * 1e-3) / 1e9, "peak": hbm_peak, "unit": "GB/s"}
    step_roof["frac"] = step_roof["achieved"] / hbm_peak

    # the paper's batch scheme on the device: b_s = 1e8-pair buffers on 3 streams, sized
    # by the 1 % estimator, each batch copied into the caller's HBM buffer -- the same step with
    # the in-place fast path switched off
    batched = None
    if args.batched_steps > 0:
        def step_batched():
            h = build()
            h.set_option("fast_path", 0)
            rc, c = h.self_join(out, cap)
            st = h.stats()
            h.close()
            return rc, c, st
        step_batched()
        torch.cuda.synchronize()
        bms, nbat = [], 0
        for i in range(args.batched_steps):
            flush_buf.fill_(i & 0xFF)
            torch.cuda.synchronize()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            rc, c, stb = step_batched()
            b.record(stream)
            torch.cuda.synchronize()
            assert rc == sj.SJ_OK and c == local_pairs
            bms.append(a.elapsed_time(b))
            nbat = stb["batches"]
        b_ms = sum(bms)
        if world > 1:
            b_ms = sjdist.allreduce_counts([int(b_ms * 1e6)], group, dev, op=dist.ReduceOp.MAX)[0] / 1e6
        batched = {"value": d_alg * args.batched_steps / (b_ms * 1e-3), "unit": "calcs/s",
                   "ms_per_step": b_ms / args.batched_steps, "steps": args.batched_steps, "batches": nbat,
                   "batch_pairs": 100_000_000, "streams": 3,
                   "note": "P:71 batch scheme on the device (fast path off): estimator-sized b_s buffers, D2D copies"}

    # e2e: the same step through the C ABI from pinned host buffers (H2D + D2H inside)
    e2e = None
    if args.e2e_steps > 0:
        h_pts = torch.from_numpy(pts).pin_memory()
        h_out = torch.empty((cap, 2), dtype=torch.int32, pin_memory=True)

        def step_host():
            if world == 1:
                h = sj.Handle(h_pts, cfg.eps, k=k)
            elif args.mp == "replicated":
                h = sj.Handle(h_pts, cfg.eps, k=k)
                h.set_slice(rank, world)
            else:
                h = sj.Handle(h_pts, cfg.eps, k=k) if rank == 0 else None
                h, _ = sjdist.replicate_index(h, 0, group, dev)
                h.set_option("k", k)
                h.set_slice(rank, world)
            rc, c = h.self_join(h_out, cap)
            h.close()
            if world > 1:
                sjdist.allreduce_counts([c], group, dev)
            return rc, c

        step_host()
        step_host()  # the first staged joins grow the memory pool and pin the slot buffers
        torch.cuda.synchronize()
        es = []
        for i in range(args.e2e_steps):
            flush_buf.fill_(i & 0xFF)
            torch.cuda.synchronize()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            rc, c = step_host()
            b.record(stream)
            torch.cuda.synchronize()
            assert rc == sj.SJ_OK and c == local_pairs
            es.append(a.elapsed_time(b))
        e_ms = sum(es)
        if world > 1:
            e_ms = sjdist.allreduce_counts([int(e_ms * 1e6)], group, dev, op=dist.ReduceOp.MAX)[0] / 1e6
        e2e = {"value": d_alg * args.e2e_steps / (e_ms * 1e-3), "unit": "calcs/s",
               "h2d_bytes_per_step": int(pts.nbytes) if (world == 1 or rank == 0) else 0,
               "d2h_bytes_per_step": int(local_pairs * 8), "ms_per_step": e_ms / args.e2e_steps,
               "steps": args.e2e_steps, "ms_min": min(es)}
        # against the measured PCIe rates: the time the step's copies need at the link's speed
        rates = pcie_rates(dev)
        t_link = e2e["h2d_bytes_per_step"] / rates["h2d"] + e2e["d2h_bytes_per_step"] / rates["d2h"]
        e2e["pcie"] = {"h2d_gbs": rates["h2d"] / 1e9, "d2h_gbs": rates["d2h"] / 1e9,
                       "copy_ms_at_link_rate": t_link * 1e3, "frac": t_link / (e2e["ms_per_step"] * 1e-3)}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = oracle_baseline(pts, cfg.eps, d_alg, args.ref_stride)
        one = oracle_baseline(pts, cfg.eps, d_alg, 0, budget_s=8.0, threads=1)
        cpu["one_core"] = {"value": one["value"], "unit": "calcs/s", "cores": 1, "sample": one["sample"]}
        cpu["o1_bruteforce_c1"] = o1_c1_timing()
        cpu.pop("seconds", None)
        cpu.pop("stride", None)

    if rank == 0:
        line = {
            "metric": "distance calcs/s", "value": value, "unit": "calcs/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": total_ms / args.steps, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic, seeded (workloads/, SURVEY.md §8.0 recipe)",
            "config": {"workload": f"{cfg.name}: {cfg.note}", "n": cfg.n, "dim": cfg.dim, "eps": cfg.eps, "k": k,
                       "pairs": tot_pairs, "dist_calcs": d_alg, "n_cells": st0["n_cells"],
                       "fwd_runs": st0["fwd_runs"], "parallelism": f"{args.mp} index + queue slices x{world}" if world > 1 else "1 GPU",
                       "l2": "flushed before every step (256 MiB write, outside the step events)",
                       "output": "HBM-resident pairs (uint32 x2), written in place"},
            "self_join_s": total_ms / args.steps / 1e3,
            "ms_per_step_median": statistics.median(step_ms), "ms_per_step_min": step_sorted[0],
            "ms_per_step_max": step_sorted[-1],
            "phases_ms": {"build": statistics.mean(build_ms), "estimate": statistics.mean(est_ms),
                          "join": mean_join_ms, "step": total_ms / args.steps,
                          "join_min": min(join_ms), "join_max": max(join_ms),
                          "join_median": statistics.median(join_ms), "build_median": statistics.median(build_ms),
                          "step_min": min(step_ms), "step_max": max(step_ms)},
            "roofline": roof,
            "build_roofline": build_roof,
            "step_roofline": step_roof,
            "batched": batched,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": int(launches),
            "clocks": clocks,
        }
        if "wee" in facts:
            line["warp_exec_efficiency"] = {"value": facts["wee"], "source": facts.get("source"),
                                            "measured": facts.get("measured"),
                                            "kind": "ncu smsp__thread_inst_executed_per_inst_executed / 32, "
                                                    "this config's emitting join launch, separate process"}
        emit(line, args)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
