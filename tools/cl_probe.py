"""Cluster-per-matrix classes (csrc/bqr_cl.cuh) against the default class:
parity of geqrf and the fused Q^H b against the fp64 oracle, and kernel time
(CUDA events, after the bench's 256 MB L2 flush) at several batches of the
STAP shape 240 x 66 c64.  Each variant runs in its own process
(BQR_FORCE_VARIANT is read once per process).

    python tools/cl_probe.py [default alt_cl4_c64_256x72_aug alt_cl2_c64_256x72_aug]
    CL_PROBE_LIB=abl/libbqr_X.so python tools/cl_probe.py ...   (an experiment build)
"""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
variants = sys.argv[1:] or ["default", "alt_cl4_c64_256x72_aug", "alt_cl2_c64_256x72_aug"]
for var in variants:
    code = f"""
import sys, json, ctypes; sys.path.insert(0, {ROOT!r}); sys.path.insert(0, {os.path.join(ROOT, 'tests')!r})
import torch, numpy as np
import os
import paper_conf_ipps_andersonsk12_b200 as bqr
if os.environ.get('CL_PROBE_LIB'):
    bqr._LIB_PATH = os.path.abspath(os.environ['CL_PROBE_LIB'])
import bqr_inputs
from oracle.compare import compare_geqrf, compare_apply
from gpu_util import geqrf_gpu, geqrf_qhb_gpu
var = {var!r}
lib = bqr.load()
row = {{'variant': var, 'lib': os.environ.get('CL_PROBE_LIB', 'in-tree'), 'kernel': bqr.kernel_name(bqr.C64, 240, 66),
       'qhb_kernel': lib.bqr_qhb_kernel_name(bqr.C64, 240, 66, 1).decode()}}
par = []
for (m, n, b, seed) in ((240, 66, 5, 1), (240, 66, 37, 2), (256, 72, 3, 3), (200, 50, 4, 4), (97, 13, 3, 5)):
    A = bqr_inputs.random_batch(m, n, b, 'c64', seed=seed)
    out, tau = geqrf_gpu(A, m)
    rep = compare_geqrf(A, m, out, tau, full_q=False)
    par.append(dict(shape=[m, n, b], ok=bool(rep['ok']), resid=float(rep['residual_max'])))
A = bqr_inputs.random_batch(240, 66, 9, 'c64', seed=6)
B = bqr_inputs.rhs_batch(240, 1, 9, 'c64', seed=6)
out, tau, QhB = geqrf_qhb_gpu(A, 240, B)
r1 = compare_geqrf(A, 240, out, tau, full_q=False)
r2 = compare_apply(out, 240, 66, tau, B, QhB)
par.append(dict(shape='qhb 240x66+1 x9', ok=bool(r1['ok'] and r2['ok'])))
row['parity'] = par
row['parity_ok'] = all(p['ok'] for p in par)
big = torch.empty(256 << 20, dtype=torch.uint8, device='cuda')
times = {{}}
for b in (1, 16, 32, 37, 64, 74, 148, 256):
    A0 = torch.randn(b, 66, 240, dtype=torch.complex64, device='cuda')
    A = torch.empty_like(A0)
    tau = torch.empty(b, 66, dtype=torch.complex64, device='cuda')
    s = torch.cuda.current_stream()
    ts = []
    for it in range(13):
        A.copy_(A0)
        if not os.environ.get('CL_PROBE_NOFLUSH'):
            big.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        st = bqr.geqrf_batched_ptr(bqr.C64, 240, 66, b, A.data_ptr(), 240, tau.data_ptr(), s.cuda_stream)
        e1.record(s)
        torch.cuda.synchronize()
        assert st == 0, st
        if it >= 3:
            ts.append(e0.elapsed_time(e1) * 1e3)
    times[b] = round(sorted(ts)[len(ts) // 2], 2)
row['geqrf_us_noflush' if os.environ.get('CL_PROBE_NOFLUSH') else 'geqrf_us_flushed'] = times
# the C4 bench step: fused geqrf + Q^H b (one right-hand side) at batch 256
b = 256
A0 = torch.randn(b, 66, 240, dtype=torch.complex64, device='cuda')
B0 = torch.randn(b, 1, 240, dtype=torch.complex64, device='cuda')
A, Bm = torch.empty_like(A0), torch.empty_like(B0)
tau = torch.empty(b, 66, dtype=torch.complex64, device='cuda')
s = torch.cuda.current_stream()
ts = []
for it in range(13):
    A.copy_(A0); Bm.copy_(B0)
    big.zero_()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    st = lib.bqr_geqrf_qhb_batched(bqr.C64, 240, 66, 1, b, ctypes.c_void_p(A.data_ptr()), 240,
                                   ctypes.c_void_p(tau.data_ptr()), ctypes.c_void_p(Bm.data_ptr()), 240,
                                   ctypes.c_void_p(s.cuda_stream))
    e1.record(s)
    torch.cuda.synchronize()
    assert st == 0, st
    if it >= 3:
        ts.append(e0.elapsed_time(e1) * 1e3)
row['qhb_256_us_flushed'] = round(sorted(ts)[len(ts) // 2], 2)
print(json.dumps(row), flush=True)
"""
    env = dict(os.environ)
    if var != "default":
        env["BQR_FORCE_VARIANT"] = var
    subprocess.run([sys.executable, "-c", code], check=False, env=env, timeout=600)
