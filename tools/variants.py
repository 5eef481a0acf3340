"""Time every registered variant of one config (kernel-only, L2 flushed).

    python tools/variants.py C3 name1 name2 ...
Prints one JSON line per variant; parity of each variant is checked on the
first 64 matrices against the oracle."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
cfg = sys.argv[1]
names = sys.argv[2:]
for nm in names:
    env = dict(os.environ, BQR_FORCE_VARIANT=nm)
    code = f"""
import sys, json; sys.path.insert(0, {ROOT!r}); sys.path.insert(0, {os.path.join(ROOT, 'tests')!r})
import os, torch, bench, numpy as np
import paper_conf_ipps_andersonsk12_b200 as bqr
import bqr_inputs
from oracle.compare import compare_geqrf
from gpu_util import geqrf_gpu
c = bqr_inputs.CONFIGS[{cfg!r}]
A = bqr_inputs.config_batch({cfg!r}, stop=64)
out, tau = geqrf_gpu(A, c['m'])
rep = compare_geqrf(A, c['m'], out, tau, full_q=c['m'] <= 128)
w = bench.Workload({cfg!r}, 0, 1, torch, bqr)
flush = torch.empty(256 << 20, dtype=torch.uint8, device='cuda')
class A_: pass
smp = bench.ClockSampler(0, 0.005)
s_ms, q_ms = bench.time_workload(w, 50, 5, torch, None, 1, flush, sampler=smp, fused=bool(int(os.environ.get('FUSED', '0'))))
clk = smp.summary()
print(json.dumps({{'variant': {nm!r}, 'kernel': bqr.kernel_name(w.code, w.m, w.n), 'qr_us': round(q_ms*1e3, 2),
   'step_us': round(s_ms*1e3, 2), 'gflops': round(w.flops/(q_ms/1e3)/1e9, 1), 'parity_ok': rep['ok'],
   'resid': rep['residual_max'], 'orth': rep['orth_max'], 'sm_mhz': clk['sm_mhz'], 'reasons': clk['reasons']}}))
"""
    r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True)
    print(r.stdout.strip() or r.stderr[-2000:], flush=True)
