"""Attribute ncu per-instruction counts (executed instructions, stall
samples) of one kernel to the source functions of its inline call chain.

    python tools/sass_attrib.py <cubin> <kernel-mangled-name> <ncu source csv(.gz)> <source.cuh>

The SASS offsets come from `nvdisasm -gi` (line info with inline chains,
needs -lineinfo); each instruction is charged to every distinct function of
<source.cuh> on its chain (so a callee's cost also shows in its callers) and
to its innermost function alone ("self")."""
import csv
import gzip
import io
import re
import subprocess
import sys
from collections import defaultdict

cubin, kname, csvp, srcp = sys.argv[1:5]
dis = subprocess.run(["nvdisasm", "-gi", cubin], capture_output=True, text=True).stdout
lines = dis.splitlines()
start = None
for i, l in enumerate(lines):
    if l.startswith(".text." + kname + ":"):
        start = i
        break
assert start is not None, kname
chain = []
off2chain = {}
pend = []
for l in lines[start + 1:]:
    if l.startswith(".L_x_") and "//" not in l and l.rstrip().endswith(":"):
        continue
    if l.startswith("//---") or l.startswith("\t.section"):
        break
    m = re.match(r"\s*//## File \"([^\"]+)\", line (\d+)(?: inlined at \"([^\"]+)\", line (\d+))?", l)
    if m:
        pend.append((m.group(1), int(m.group(2)), m.group(3), int(m.group(4)) if m.group(4) else None))
        continue
    m = re.match(r"\s*/\*([0-9a-f]{4,})\*/\s+(.*)", l)
    if m:
        if pend:
            chain = [(f, ln) for f, ln, _, _ in pend]
            pend = []
        off2chain[int(m.group(1), 16)] = list(chain)

# function line ranges of the source
src = open(srcp).read().splitlines()
funcs = []
for i, l in enumerate(src, 1):
    m = re.match(r"^(?:__global__ void .*?|__device__ __forceinline__ [\w:<>,\s&*]+?)\s(\w+)\s*\(", l)
    if m:
        funcs.append((i, m.group(1)))
def fn_of(ln):
    name = "?"
    for s, n in funcs:
        if s <= ln:
            name = n
    return name

op = gzip.open if csvp.endswith(".gz") else open
rows = list(csv.reader(io.TextIOWrapper(op(csvp, "rb"))))
hdr = rows[1]
ix = {h: i for i, h in enumerate(hdr)}
base = int(rows[2][ix["Address"]], 16)
stc = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
reasons = defaultdict(lambda: defaultdict(int))
incl = defaultdict(lambda: [0, 0])
self_ = defaultdict(lambda: [0, 0])
tot = [0, 0]
for r in rows[2:]:
    try:
        off = int(r[ix["Address"]], 16) - base
    except ValueError:
        continue
    ex = int(r[ix["Instructions Executed"]] or 0)
    sm = int(r[ix["Warp Stall Sampling (All Samples)"]] or 0)
    tot[0] += ex
    tot[1] += sm
    ch = off2chain.get(off, [])
    names = []
    for f, ln in ch:
        if f.endswith(srcp.split("/")[-1]):
            nm = f"{fn_of(ln)}"
            if nm not in names:
                names.append(nm)
    inner = names[0] if names else "?"
    self_[inner][0] += ex
    self_[inner][1] += sm
    for nm in names:
        incl[nm][0] += ex
        incl[nm][1] += sm
        for h in stc:
            reasons[nm][h[6:]] += int(r[ix[h]] or 0)
    # outer call line (caller context)
    outer = [ln for f, ln in ch if f.endswith(srcp.split("/")[-1])]
    if outer:
        key = f"{fn_of(outer[-1])}:{outer[-1]} <- ... {inner}"
print(f"total executed {tot[0]}  samples {tot[1]}")
print("%-22s %12s %7s %8s %7s" % ("function (inclusive)", "exec", "exec%", "samples", "samp%"))
for k, (e, s) in sorted(incl.items(), key=lambda kv: -kv[1][1]):
    print("%-22s %12d %6.1f%% %8d %6.1f%%" % (k, e, 100 * e / tot[0], s, 100 * s / max(1, tot[1])))
print("stall reasons (inclusive):")
for k, (e, s_) in sorted(incl.items(), key=lambda kv: -kv[1][1]):
    rs = reasons[k]
    tot_r = max(1, sum(rs.values()))
    print("  %-20s " % k + " ".join(f"{n}={100 * v / tot_r:.0f}%" for n, v in sorted(rs.items(), key=lambda kv: -kv[1])[:7]))
print("%-22s %12s %7s %8s %7s" % ("function (self)", "exec", "exec%", "samples", "samp%"))
for k, (e, s) in sorted(self_.items(), key=lambda kv: -kv[1][1]):
    print("%-22s %12d %6.1f%% %8d %6.1f%%" % (k, e, 100 * e / tot[0], s, 100 * s / max(1, tot[1])))
