"""A/B of dispatch variants in one build (BQR_FORCE_VARIANT per process):
geqrf kernel time for one config (bench.time_workload, L2 flushed) plus a
parity check of sampled matrices against the fp64 oracle (odd batch, full
batch every 97th matrix).

    python tools/variant_ab.py C3 default alt_rf_f32_R4G4_14x14_x2_exact
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
cfg = sys.argv[1]
for var in sys.argv[2:]:
    code = f"""
import sys; sys.path.insert(0, {ROOT!r}); sys.path.insert(0, {os.path.join(ROOT, 'tests')!r})
import numpy as np
import paper_conf_ipps_andersonsk12_b200 as bqr
import torch, bench, json, bqr_inputs
from oracle.compare import compare_geqrf
from gpu_util import geqrf_gpu
c = bqr_inputs.CONFIGS[{cfg!r}]
m, n = c['m'], c['n']
name = bqr.kernel_name(bqr.R32 if c['dtype'] == 'f32' else bqr.C64, m, n)
reps = []
A = bqr_inputs.random_batch(m, n, 33, c['dtype'], c['seed'], c['dist'])
out, tau = geqrf_gpu(A, m)
reps.append(compare_geqrf(A, m, out, tau, full_q=m <= 128))
A = bqr_inputs.config_batch({cfg!r})
out, tau = geqrf_gpu(A, m)
idx = np.arange(0, A.shape[0], 97)
reps.append(compare_geqrf(A[idx], m, out[idx], tau[idx], full_q=m <= 128))
w = bench.Workload({cfg!r}, 0, 1, torch, bqr)
flush = torch.empty(256 << 20, dtype=torch.uint8, device='cuda')
smp = bench.ClockSampler(0, 0.005)
s_ms, q_ms = bench.time_workload(w, 50, 5, torch, None, 1, flush, sampler=smp, fused=False)
print(json.dumps({{'cfg': {cfg!r}, 'variant': {var!r}, 'kernel': name, 'qr_us': round(q_ms * 1e3, 2),
                  'gflops': round(w.flops / q_ms / 1e6, 1), 'parity_ok': all(r['ok'] for r in reps),
                  'resid': max(r['residual_max'] for r in reps), 'orth': max(r['orth_max'] for r in reps),
                  'sm_mhz': smp.summary()['sm_mhz']}}))
"""
    env = dict(os.environ)
    env.pop("BQR_FORCE_VARIANT", None)
    if var != "default":
        env["BQR_FORCE_VARIANT"] = var
    r = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, env=env)
    print(r.stdout.strip() or r.stderr[-2500:], flush=True)
