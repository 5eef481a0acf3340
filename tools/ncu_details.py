"""Key metrics of the first kernel in an ncu report (details page)."""
import csv
import io
import subprocess
import sys

WANT = ["Duration", "Elapsed Cycles", "SM Frequency", "Executed Ipc Active", "Issue Slots Busy",
        "Executed Instructions", "Warp Cycles Per Issued Instruction", "Eligible Warps Per Scheduler",
        "Achieved Active Warps Per SM", "Registers Per Thread", "Grid Size", "Block Size",
        "Dynamic Shared Memory Per Block", "DRAM Throughput", "Memory Throughput", "L2 Hit Rate",
        "Compute (SM) Throughput", "Theoretical Occupancy", "Avg. Active Threads Per Warp",
        "Local Memory Spilling Requests"]
out = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "details", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = rows[0]
idx = {h: i for i, h in enumerate(hdr)}
seen = set()
for r in rows[1:]:
    if r[idx["ID"]] != "0":
        continue
    n = r[idx["Metric Name"]]
    if n in WANT and n not in seen:
        seen.add(n)
        print(f"{n:40s} {r[idx['Metric Value']]} {r[idx['Metric Unit']]}")
