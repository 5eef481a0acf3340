"""Per-instruction stall analysis of an ncu source-page CSV (gz ok):
top instructions for a given stall column, and stall totals by opcode."""
import csv, gzip, io, sys, collections

path, col = sys.argv[1], sys.argv[2]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 25
f = gzip.open(path, "rt") if path.endswith(".gz") else open(path)
rows = list(csv.reader(f))
hdr = rows[1]
ix = {h: i for i, h in enumerate(hdr)}
data = rows[2:]
c = ix[col]
tot = sum(float(r[c] or 0) for r in data)
print(f"{col}: total {tot:.0f} samples over {len(data)} instructions")
by_op = collections.Counter()
for r in data:
    op = r[ix["Source"]].split()[0] if r[ix["Source"]].split() else "?"
    if op.startswith("@"):
        op = r[ix["Source"]].split()[1]
    by_op[op.split(".")[0]] += float(r[c] or 0)
print("by opcode:", ", ".join(f"{k} {v:.0f}" for k, v in by_op.most_common(12)))
idx = sorted(range(len(data)), key=lambda i: -float(data[i][c] or 0))[:top]
for i in sorted(idx):
    r = data[i]
    print(f"{i:6d} {float(r[c] or 0):6.0f}  exec {r[ix['Instructions Executed']]:>8s}  {r[ix['Source']].strip()[:90]}")
