"""A/B timing of two builds of libbqr.so (same box, same call): geqrf-only
kernel time for one config, via BQR_LIB override.

    python tools/ab_lib.py C4 oldlib/libbqr_X.so paper_conf_ipps_andersonsk12_b200/libbqr.so
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
cfg = sys.argv[1]
for lib in sys.argv[2:]:
    code = f"""
import sys; sys.path.insert(0, {ROOT!r})
import paper_conf_ipps_andersonsk12_b200 as bqr
bqr._LIB_PATH = {os.path.abspath(lib)!r}
import torch, bench, json
w = bench.Workload({cfg!r}, 0, 1, torch, bqr)
flush = torch.empty(256 << 20, dtype=torch.uint8, device='cuda')
smp = bench.ClockSampler(0, 0.005)
s_ms, q_ms = bench.time_workload(w, 50, 5, torch, None, 1, flush, sampler=smp, fused=False)
print(json.dumps({{'lib': {lib!r}, 'qr_us': round(q_ms * 1e3, 2), 'sm_mhz': smp.summary()['sm_mhz']}}))
"""
    r = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True)
    print(r.stdout.strip() or r.stderr[-1500:], flush=True)
