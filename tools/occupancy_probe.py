"""Tail / occupancy probe for the persistent register-file kernels: kernel
time (CUDA events, L2 flushed, median of 15) of one shape at several batch
sizes and resident-CTA caps (BQR_MAX_BPS is read once per process, so each
cap runs in its own process).

    python tools/occupancy_probe.py f32 56 56 5000,4736,2368 [cap]
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import bqr_inputs  # noqa: E402
import paper_conf_ipps_andersonsk12_b200 as bqr  # noqa: E402

dt, m, n = sys.argv[1], int(sys.argv[2]), int(sys.argv[3])
batches = [int(x) for x in sys.argv[4].split(",")]
code = bqr.C64 if dt == "c64" else bqr.R32
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
s = torch.cuda.current_stream()
for B in batches:
    A = bqr_inputs.random_batch(m, n, B, dt, seed=5)
    pristine = torch.from_numpy(A).cuda()
    buf = torch.empty_like(pristine)
    tau = torch.empty((B, min(m, n)), dtype=buf.dtype, device="cuda")
    ts = []
    for it in range(18):
        buf.copy_(pristine)
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        st = bqr.geqrf_batched_ptr(code, m, n, B, buf.data_ptr(), m, tau.data_ptr(), s.cuda_stream)
        e1.record(s)
        assert st == 0
        torch.cuda.synchronize()
        if it >= 3:
            ts.append(e0.elapsed_time(e1) * 1e3)
    ts.sort()
    print(json.dumps({"dt": dt, "m": m, "n": n, "batch": B, "cap": os.environ.get("BQR_MAX_BPS", "-"),
                      "kernel": bqr.kernel_name(code, m, n), "us_median": round(ts[len(ts) // 2], 2),
                      "us_min": round(ts[0], 2)}), flush=True)
