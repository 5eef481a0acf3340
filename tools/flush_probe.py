"""Kernel time of a bench config after the bench's 256 MB write flush, a
256 MB read, a 1 MB write, and nothing (CUDA events around the geqrf launch).

    python tools/flush_probe.py S80 C2 C4
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_ipps_andersonsk12_b200 as bqr  # noqa: E402

big = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
small = torch.empty(1 << 20, dtype=torch.uint8, device="cuda")
sink = torch.empty(1, dtype=torch.float32, device="cuda")
flushes = {"write256MB": lambda: big.zero_(), "read256MB": lambda: sink.copy_(big.view(torch.float32).sum().reshape(1)),
           "write1MB": lambda: small.zero_(), "none": lambda: None}
for cfg in sys.argv[1:]:
    w = bench.Workload(cfg, 0, 1, torch, bqr)
    row = {"cfg": cfg}
    for name, fl in flushes.items():
        ts = []
        for it in range(23):
            w.restore()
            fl()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(w.stream)
            w.geqrf()
            e1.record(w.stream)
            torch.cuda.synchronize()
            if it >= 3:
                ts.append(e0.elapsed_time(e1) * 1e3)
        row[name + "_us"] = round(sorted(ts)[len(ts) // 2], 2)
    print(json.dumps(row), flush=True)
