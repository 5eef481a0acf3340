"""A/B timing of several builds of libbqr.so (same box, same call): geqrf-only
kernel time for one config, via a per-process library override, plus a
parity check of the first 32 matrices against the fp64 oracle.

    python tools/ab_lib.py C4 abl/libbqr_X.so paper_conf_ipps_andersonsk12_b200/libbqr.so
    python tools/ab_lib.py f32:128 abl/libbqr_X.so ...     (C5 cell, 4 waves of 148)
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
cfg = sys.argv[1]
for lib in sys.argv[2:]:
    code = f"""
import sys; sys.path.insert(0, {ROOT!r}); sys.path.insert(0, {os.path.join(ROOT, 'tests')!r})
import paper_conf_ipps_andersonsk12_b200 as bqr
bqr._LIB_PATH = {os.path.abspath(lib)!r}
import torch, bench, json, bqr_inputs
cfg = {cfg!r}
if ':' in cfg:
    dt, n = cfg.split(':')
    c = bqr_inputs.c5_config(int(n), dt)
    c['batch'] = 148 * 4
    bqr_inputs.CONFIGS[cfg] = c
from oracle.compare import compare_geqrf
from gpu_util import geqrf_gpu
c = bqr_inputs.CONFIGS[cfg]
A = bqr_inputs.random_batch(c['m'], c['n'], 32, c['dtype'], c['seed'], c['dist'])
out, tau = geqrf_gpu(A, c['m'])
rep = compare_geqrf(A, c['m'], out, tau, full_q=c['m'] <= 128)
w = bench.Workload(cfg, 0, 1, torch, bqr)
flush = torch.empty(256 << 20, dtype=torch.uint8, device='cuda')
smp = bench.ClockSampler(0, 0.005)
s_ms, q_ms = bench.time_workload(w, 50, 5, torch, None, 1, flush, sampler=smp, fused=False)
print(json.dumps({{'cfg': cfg, 'lib': {lib!r}, 'qr_us': round(q_ms * 1e3, 2), 'gflops': round(w.flops / q_ms / 1e6, 1),
                  'parity_ok': rep['ok'], 'resid': rep['residual_max'], 'orth': rep['orth_max'],
                  'sm_mhz': smp.summary()['sm_mhz']}}))
"""
    r = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True)
    print(r.stdout.strip() or r.stderr[-1500:], flush=True)
