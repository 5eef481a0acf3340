"""Per-loop SASS op counts of one kernel (cuobjdump -sass text on stdin):
each backward branch defines a loop body [target, branch]."""
import re
import sys
from collections import Counter

lines = sys.stdin.read().splitlines()
ins = []
for ln in lines:
    m = re.match(r"\s+/\*([0-9a-f]{4,})\*/\s+(.*?);", ln)
    if m:
        ins.append((int(m.group(1), 16), m.group(2).strip()))
addr = [a for a, _ in ins]
loops = []
for a, t in ins:
    m = re.search(r"BRA(?:\.U)?(?:\.ANY)?\s+0x([0-9a-f]+)", t)
    if m and "BRA.DIV" not in t:
        tgt = int(m.group(1), 16)
        if tgt < a:
            loops.append((tgt, a))
def op(t):
    t = re.sub(r"^@!?U?P\w+\s+", "", t)
    return t.split()[0].split(".")[0] if t else ""
print(f"total {len(ins)} instructions")
for lo, hi in loops:
    body = [t for a, t in ins if lo <= a <= hi]
    c = Counter(op(t) for t in body)
    top = ", ".join(f"{k}:{v}" for k, v in c.most_common(12))
    print(f"loop {lo:#06x}-{hi:#06x}: {len(body)} instr | {top}")
