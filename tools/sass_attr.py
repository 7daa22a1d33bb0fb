"""Attribute an ncu source-page export (per-SASS-instruction executed instructions and stall
samples) to CUDA source lines through the cubin's inline line table (nvdisasm -gi).

    python tools/sass_attr.py OBJ_OR_CUBIN FUNC_SUBSTR NCU_SASS_CSV [--depth D] [--top N]

Each instruction's inline chain (outermost call site first) is cut to D levels; rows print the
instruction share, the stall-sample share and the source text of the innermost line kept.
Diagnostic tool (profiles/ summaries)."""
import argparse
import collections
import csv
import os
import re
import subprocess
import tempfile


def sass_lines(obj, func):
    with tempfile.TemporaryDirectory() as td:
        if obj.endswith(".o") or obj.endswith(".so"):
            subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(obj)], cwd=td, check=True,
                           capture_output=True)
            cub = [os.path.join(td, f) for f in os.listdir(td) if f.endswith(".cubin")]
        else:
            cub = [obj]
        for c in cub:
            txt = subprocess.run(["nvdisasm", "-gi", "-c", c], capture_output=True, text=True).stdout
            m = re.search(r"^(\S*" + re.escape(func) + r"\S*):\s*$", txt, re.M)
            if m:
                return txt[m.end():], m.group(1)
    raise SystemExit(f"function {func} not found")


def chains(text):
    """offset -> inline chain [(file, line), ...] outermost first."""
    out = {}
    pend, last = [], []
    for ln in text.splitlines():
        if ln.startswith(".text.") or ln.startswith("\t.section"):
            break
        m = re.match(r'\s*//## File "([^"]+)", line (\d+)(?: inlined at "([^"]+)", line (\d+))?', ln)
        if m:
            pend.append((os.path.basename(m.group(1)), int(m.group(2))))
            continue
        m = re.match(r"\s*/\*([0-9a-f]{4,})\*/", ln)
        if m:
            if pend:
                # the block lists innermost first ... outermost last
                cur = list(reversed(pend))
                pend = []
                last = cur
            out[int(m.group(1), 16)] = last
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("obj")
    ap.add_argument("func")
    ap.add_argument("csv")
    ap.add_argument("--depth", type=int, default=2)
    ap.add_argument("--top", type=int, default=40)
    a = ap.parse_args()
    text, full = sass_lines(a.obj, a.func)
    ch = chains(text)
    rows = list(csv.reader(open(a.csv)))
    hdr = rows[1]
    ia, ie, iss = hdr.index("Address"), hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)")
    data = rows[2:]
    base = int(data[0][ia], 16)
    agg_i, agg_s = collections.Counter(), collections.Counter()
    tot_i = tot_s = 0
    for r in data:
        off = int(r[ia], 16) - base
        ni, ns = float(r[ie] or 0), float(r[iss] or 0)
        c = ch.get(off, [])
        key = tuple(c[: a.depth]) if c else (("?", 0),)
        agg_i[key] += ni
        agg_s[key] += ns
        tot_i += ni
        tot_s += ns
    srcs = {}
    print(f"{full[:100]}\n{int(tot_i)} warp instructions, {int(tot_s)} stall samples")
    print(f"{'instr%':>7} {'stall%':>7}  chain")
    for key, v in sorted(agg_i.items(), key=lambda kv: -agg_s[kv[0]])[: a.top]:
        f, l = key[-1]
        path = os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", "paper_conf_ipps_galletg19_b200", "csrc", f)
        if f not in srcs and os.path.exists(path):
            srcs[f] = open(path).read().splitlines()
        src = srcs.get(f, [""] * (l + 1))[l - 1].strip()[:70] if l else ""
        print(f"{100 * v / tot_i:7.2f} {100 * agg_s[key] / max(tot_s, 1):7.2f}  {' > '.join(str(x[1]) for x in key):24s} {src}")


if __name__ == "__main__":
    main()
