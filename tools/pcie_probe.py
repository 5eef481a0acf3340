"""Pinned host<->device copy bandwidth on the box (context for the e2e
number of bench.py): H2D alone, D2H alone, and both at once on two streams,
at the C3 step's byte counts (62.7 MB in, 63.8 MB out).

    python tools/pcie_probe.py [--out gpurun_out/pcie.json]
"""
import json, sys
import torch

nin, nout = 5000 * 56 * 56 * 4, 5000 * (56 * 56 + 56) * 4
hin = torch.empty(nin, dtype=torch.uint8).pin_memory()
hout = torch.empty(nout, dtype=torch.uint8).pin_memory()
din = torch.empty(nin, dtype=torch.uint8, device="cuda")
dout = torch.empty(nout, dtype=torch.uint8, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()


def timed(fn, reps=10):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ts = []
    for _ in range(reps):
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    ts.sort()
    return ts[len(ts) // 2]


def both():
    cur = torch.cuda.current_stream()
    e = torch.cuda.Event()
    e.record(cur)
    s1.wait_event(e)
    s2.wait_event(e)
    with torch.cuda.stream(s1):
        din.copy_(hin, non_blocking=True)
    with torch.cuda.stream(s2):
        hout.copy_(dout, non_blocking=True)
    cur.wait_stream(s1)
    cur.wait_stream(s2)


r = {}
t = timed(lambda: din.copy_(hin, non_blocking=True))
r["h2d_ms"], r["h2d_gbs"] = t, nin / t / 1e6
t = timed(lambda: hout.copy_(dout, non_blocking=True))
r["d2h_ms"], r["d2h_gbs"] = t, nout / t / 1e6
t = timed(both)
r["both_ms"], r["both_gbs_total"] = t, (nin + nout) / t / 1e6
r["bytes_in"], r["bytes_out"] = nin, nout
print(json.dumps(r))
if "--out" in sys.argv:
    with open(sys.argv[sys.argv.index("--out") + 1], "w") as f:
        json.dump(r, f)
