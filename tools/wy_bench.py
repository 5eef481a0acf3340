"""Compact-WY blocked QR (tensor-core trailing updates) vs the default
bqr_geqrf_batched path on the C5 complex cells beyond one SM: kernel-only
time (CUDA events, L2 flushed), useful GFLOP/s, roofline fraction, parity
on a sample against the fp64 oracle.

    python tools/wy_bench.py [n ...]
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import bqr_inputs  # noqa: E402
import bqr_metrics as bm  # noqa: E402
import paper_conf_ipps_andersonsk12_b200 as bqr  # noqa: E402
from oracle.compare import compare_geqrf  # noqa: E402

args = sys.argv[1:]
cells = []
for a in args or ["c64:176", "c64:192", "c64:224", "c64:256"]:
    dt, n = (a.split(":") if ":" in a else ("c64", a))
    cells.append((dt, int(n)))
n_sm = torch.cuda.get_device_properties(0).multi_processor_count
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
peaks = bm.load_peaks()
for dt, n in cells:
    code = bqr.C64 if dt == "c64" else bqr.R32
    cfg = bqr_inputs.c5_config(n, dt, n_sm=n_sm)
    B = cfg["batch"]
    A = bqr_inputs.random_batch(n, n, B, dt, cfg["seed"])
    pristine = torch.from_numpy(A).cuda()
    buf = torch.empty_like(pristine)
    tau = torch.empty((B, n), dtype=buf.dtype, device="cuda")
    wsb = bqr.geqrf_wy_workspace_bytes(code, n, n, n, B)
    ws = torch.empty(max(1, wsb), dtype=torch.uint8, device="cuda")
    s = torch.cuda.current_stream()

    def run(kind):
        if kind == "wy":
            st = bqr.geqrf_wy_batched_ptr(code, n, n, B, buf.data_ptr(), n, tau.data_ptr(), ws.data_ptr(), wsb)
        else:
            st = bqr.geqrf_batched_ptr(code, n, n, B, buf.data_ptr(), n, tau.data_ptr(), s.cuda_stream)
        assert st == 0, st

    flops = B * bm.geqrf_flops(n, n, dt)
    nbytes = B * bm.geqrf_bytes(n, n, dt)
    fp32 = bm.fp32_peak_tflops(n_sm, float(peaks.get("sm_max_mhz", 1965.0)))
    t_roof, bound = bm.roofline_time_s(flops, nbytes, float(peaks["hbm_gbs"]), fp32)
    for kind in ("default", "wy"):
        for _ in range(2):
            buf.copy_(pristine)
            run(kind)
        ts = []
        for _ in range(10):
            buf.copy_(pristine)
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            run(kind)
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        ms = float(np.median(ts))
        idx = np.arange(0, B, 97)
        out = buf[torch.from_numpy(idx).cuda()].cpu().numpy()
        tu = tau[torch.from_numpy(idx).cuda()].cpu().numpy()
        rep = compare_geqrf(A[idx], n, out, tu, full_q=False)
        name = bqr.load().bqr_geqrf_wy_kernel_name(code, n, n, n).decode() if kind == "wy" else bqr.kernel_name(code, n, n)
        print(json.dumps({"n": n, "dtype": dt, "batch": B, "path": kind, "kernel": name, "ms": round(ms, 4),
                          "tflops": round(flops / ms / 1e9, 3), "roofline_frac": round(t_roof / (ms / 1e3), 4),
                          "bound": bound, "parity_ok": rep["ok"], "residual": rep["residual_max"],
                          "orth": rep["orth_max"], "sampled": len(idx)}), flush=True)
