"""Run a few geqrf (+apply) launches of one config -- the command ncu wraps.

    python tools/run_once.py C3 [reps]
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_ipps_andersonsk12_b200 as bqr  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C3"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
torch.cuda.set_device(0)
w = bench.Workload(name, 0, 1, torch, bqr)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for _ in range(reps):
    w.restore()
    flush.zero_()
    if w.nrhs and w.kind == "qr":
        w.geqrf_qhb()  # the bench step: fused factorisation + Q^H b
    else:
        w.geqrf()
torch.cuda.synchronize()
print("done", name, bqr.kernel_name(w.code, w.m, w.n))
