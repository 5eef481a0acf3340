"""Per-column chain of the cluster-per-matrix kernel (debug build with
-DBQR_CL_TIMING; stamps of the look-ahead owner, first matrix): cycles from
v_k arriving at the owner of column k+1 to its dot + update of that column,
its norm, the publication of reflector k+1, and on to v_{k+1} arriving at the
next owner.  Use the one-CTA variant (alt_cl1_*) so every stamp is on one
SM's clock.

    BQR_FORCE_VARIANT=alt_cl1_c64_256x72_aug python tools/cl_timing.py abl/libbqr_cltime.so [batch]
"""
import ctypes
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_andersonsk12_b200 as bqr  # noqa: E402

bqr._LIB_PATH = os.path.abspath(sys.argv[1])
lib = bqr.load()
batch = int(sys.argv[2]) if len(sys.argv) > 2 else 1
A0 = torch.randn(batch, 66, 240, dtype=torch.complex64, device="cuda")
A = torch.empty_like(A0)
tau = torch.empty(batch, 66, dtype=torch.complex64, device="cuda")
for _ in range(3):
    A.copy_(A0)
    assert bqr.geqrf_batched_ptr(bqr.C64, 240, 66, batch, A.data_ptr(), 240, tau.data_ptr(),
                                 torch.cuda.current_stream().cuda_stream) == 0
    torch.cuda.synchronize()
buf = np.zeros(80 * 4, dtype=np.int64)
lib.bqr_cl_debug_stamps.argtypes = [ctypes.c_void_p, ctypes.c_size_t]
assert lib.bqr_cl_debug_stamps(buf.ctypes.data_as(ctypes.c_void_p), ctypes.c_size_t(buf.nbytes)) == 0
st = buf.reshape(80, 4)[:65]
ok = (st > 0).all(axis=1)
st = st[ok]
dot = st[:, 1] - st[:, 0]
norm = st[:, 2] - st[:, 1]
pub = st[:, 3] - st[:, 2]
xfer = st[1:, 0] - st[:-1, 3]
step = st[1:, 0] - st[:-1, 0]
print(f"variant={os.environ.get('BQR_FORCE_VARIANT')} batch={batch} steps={len(st)}")
for name, x in (("v_k arrived -> dot+update col k+1", dot), ("-> norm reduced", norm),
                ("-> xLARFG + scale + publish issued", pub), ("publish issued -> next owner has v", xfer),
                ("per column (arrival to arrival)", step)):
    print(f"{name:40s} median {int(np.median(x)):6d}  mean {int(np.mean(x)):6d}  min {int(np.min(x)):6d}")
