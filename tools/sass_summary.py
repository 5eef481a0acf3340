"""Static per-kernel summary of libbqr.so (cuobjdump, no GPU): registers,
local-memory (spill) bytes, shared memory, SASS instruction count and the
counts of the mnemonics that matter for these kernels.

    python tools/sass_summary.py [regex-of-kernel-names] > profiles/r02/sass_summary.txt
"""
import collections
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "paper_conf_ipps_andersonsk12_b200", "libbqr.so")
pat = re.compile(sys.argv[1] if len(sys.argv) > 1 else
                 r"geqrf_ll56|getrf_lll56|gj_llgj56|geqrf_cl_kernel|geqrf_llc240|"
                 r"geqrf_rf_kernelI6float2Li32ELi12ELi8ELi6ELi1ELb0ELb0ELb1|geqrf_rf_kernelI6float2Li16ELi4ELi5ELi4|"
                 r"geqrf_rf_kernelI6float2Li32ELi16ELi6ELi6|geqrf_tiny_kernelIfLi4ELi4")
OPS = ["FFMA", "FFMA2", "FADD", "FMUL", "SHFL", "LDS", "STS", "LDG", "STG", "LDL", "STL", "STAS", "SYNCS",
       "MEMBAR", "UBLKCP", "UTMALDG", "UTCHMMA", "BRA"]

res = subprocess.run(["cuobjdump", "-res-usage", LIB], capture_output=True, text=True).stdout
usage = {}
fn = None
for line in res.splitlines():
    m = re.search(r"Function (\S+):", line)
    if m:
        fn = m.group(1)
        continue
    m = re.search(r"REG:(\d+) STACK:(\d+) SHARED:(\d+) LOCAL:(\d+)", line)
    if m and fn:
        usage[fn] = dict(reg=int(m.group(1)), stack=int(m.group(2)), shared=int(m.group(3)), local=int(m.group(4)))

sass = subprocess.run(["cuobjdump", "-sass", LIB], capture_output=True, text=True).stdout
counts = collections.defaultdict(collections.Counter)
fn = None
for line in sass.splitlines():
    m = re.search(r"Function : (\S+)", line)
    if m:
        fn = m.group(1)
        continue
    m = re.match(r"\s+/\*[0-9a-f]+\*/\s+(?:@!?U?P\w+\s+)?([A-Z][A-Z0-9_]*)(\.[A-Z0-9_.]+)?", line)
    if m and fn:
        counts[fn]["_total"] += 1
        op = m.group(1)
        counts[fn][op] += 1

print("# libbqr.so static kernel summary (tools/sass_summary.py; cuobjdump -res-usage / -sass, sm_100a)")
print("# kernel | regs | stack B | local B | static smem B | SASS instrs | " + " ".join(OPS))
for fn in sorted(counts):
    if not pat.search(fn):
        continue
    u = usage.get(fn, {})
    c = counts[fn]
    print(f"{fn} | {u.get('reg', '?')} | {u.get('stack', '?')} | {u.get('local', '?')} | {u.get('shared', '?')} | {c['_total']} | "
          + " ".join(f"{o}={c[o]}" for o in OPS if c[o]))
