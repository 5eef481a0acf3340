"""Kernel time vs batch size (wave quantisation / per-round latency).

    python tools/batch_scan.py C3 2 592 1184 2368 4736 5000
Prints one JSON line per batch: geqrf-only time (L2 flushed, median of 30),
matrices per round implied, and the kernel name.  BQR_FORCE_VARIANT applies.
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_ipps_andersonsk12_b200 as bqr  # noqa: E402

cfg = sys.argv[1]
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for b in [int(x) for x in sys.argv[2:]]:
    w = bench.Workload(cfg, 0, 1, torch, bqr, batch=b)
    ts = []
    for it in range(35):
        w.restore()
        flush.fill_(it & 0xff)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record(w.stream)
        w.geqrf()
        e1.record(w.stream)
        torch.cuda.synchronize()
        if it >= 5:
            ts.append(e0.elapsed_time(e1) * 1e3)
    us = float(np.median(ts))
    print(json.dumps({"cfg": cfg, "batch": b, "us": round(us, 2), "min_us": round(min(ts), 2),
                      "us_per_matrix": round(us / b, 4), "gflops": round(w.flops / us / 1e3, 1),
                      "kernel": bqr.kernel_name(w.code, w.m, w.n)}), flush=True)
