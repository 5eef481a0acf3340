"""Component times of a tiled C4 (256 x 240x66 c64 + Q^H b) with panel
width nb: geqrf of the 240 x nb panel, Q^H of its nb reflectors on the
66 - nb + 1 trailing columns, fused geqrf + Q^H b of the (240 - nb) x
(66 - nb) trailing matrix (CUDA events, L2 flushed before each call).

    python tools/tiled_probe.py 22 33
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_andersonsk12_b200 as bqr  # noqa: E402

flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
B = 256


def rnd(m, n):
    return bqr.colmajor(torch.randn(B, m, n, dtype=torch.complex64, device="cuda"))


def timed(fn, reps=20):
    ts = []
    for i in range(reps + 3):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        if i >= 3:
            ts.append(e0.elapsed_time(e1) * 1e3)
    return round(sorted(ts)[len(ts) // 2], 2)


for nb in [int(x) for x in sys.argv[1:]] or [33]:
    A1 = rnd(240, nb)
    t1 = torch.empty(B, nb, dtype=torch.complex64, device="cuda")
    bqr.geqrf_batched(A1, t1)
    C = rnd(240, 66 - nb + 1)
    A2 = rnd(240 - nb, 66 - nb)
    b2 = rnd(240 - nb, 1)
    row = {"nb": nb,
           "panel_kernel": bqr.kernel_name(bqr.C64, 240, nb),
           "panel_us": timed(lambda: bqr.geqrf_batched(A1, t1)),
           "apply_us": timed(lambda: bqr.apply_qh_batched(A1, t1, C)),
           "trail_kernel": bqr.load().bqr_qhb_kernel_name(bqr.C64, 240 - nb, 66 - nb, 1).decode(),
           "trail_us": timed(lambda: bqr.geqrf_qhb_batched(A2, b2))}
    row["sum_us"] = round(row["panel_us"] + row["apply_us"] + row["trail_us"], 2)
    print(json.dumps(row), flush=True)
Af = rnd(240, 66)
bf = rnd(240, 1)
print(json.dumps({"fused_one_kernel_us": timed(lambda: bqr.geqrf_qhb_batched(Af, bf)),
                  "kernel": bqr.load().bqr_qhb_kernel_name(bqr.C64, 240, 66, 1).decode()}))
