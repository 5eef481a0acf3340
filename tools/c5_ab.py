"""A/B of dispatch variants (BQR_FORCE_VARIANT) on one C5 cell at its bench
batch (kernel time, L2 flushed) with a sampled oracle check.

    python tools/c5_ab.py c64 56 default rf_c64_R8G8_8x8_cta
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
dt, n = sys.argv[1], int(sys.argv[2])
for var in sys.argv[3:]:
    code = f"""
import sys; sys.path.insert(0, {ROOT!r}); sys.path.insert(0, {os.path.join(ROOT, 'tests')!r})
import numpy as np, torch, json, bench, bqr_inputs
import paper_conf_ipps_andersonsk12_b200 as bqr
from oracle.compare import compare_geqrf
from gpu_util import geqrf_gpu
cfg = bqr_inputs.c5_config({n}, {dt!r})
bqr_inputs.CONFIGS['C5X'] = cfg
A = bqr_inputs.random_batch({n}, {n}, 300, {dt!r}, cfg['seed'])
out, tau = geqrf_gpu(A, {n})
rep = compare_geqrf(A, {n}, out, tau, full_q=True)
w = bench.Workload('C5X', 0, 1, torch, bqr)
flush = torch.empty(256 << 20, dtype=torch.uint8, device='cuda')
_, q = bench.time_workload(w, 20, 3, torch, None, 1, flush, fused=False)
t_roof, _ = bench.bm.roofline_time_s(w.flops, w.bytes, 6551.0, bench.bm.fp32_peak_tflops(148, 1965.0))
print(json.dumps({{'cell': '{dt} {n}', 'batch': cfg['batch'], 'variant': {var!r},
                  'kernel': bqr.kernel_name(bqr.R32 if {dt!r} == 'f32' else bqr.C64, {n}, {n}),
                  'us': round(q * 1e3, 2), 'frac': round(t_roof / (q / 1e3), 4), 'parity_ok': rep['ok']}}))
"""
    env = dict(os.environ)
    env.pop("BQR_FORCE_VARIANT", None)
    if var != "default":
        env["BQR_FORCE_VARIANT"] = var
    r = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, env=env)
    print(r.stdout.strip() or r.stderr[-2000:], flush=True)
