"""Per-column timeline of the left-looking C4 experiment (debug build with
-DBQR_LLC_TIMING, BQR_FORCE_VARIANT=alt_llc_c64_240x66_left3_aug): for CTA
0's first matrix, when each warp's wait for v_k returned and when v_{k+1}
was published.

    python tools/llc_timing.py abl/libbqr_llctime.so [batch]
"""
import ctypes
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_ipps_andersonsk12_b200 as bqr  # noqa: E402

bqr._LIB_PATH = os.path.abspath(sys.argv[1])
lib = bqr.load()
W = 6
w = bench.Workload("C4", 0, 1, torch, bqr, batch=int(sys.argv[2]) if len(sys.argv) > 2 else None)
for _ in range(3):
    w.restore()
    torch.cuda.synchronize()
    w.geqrf_qhb()
    torch.cuda.synchronize()
buf = np.zeros(W * 74 * 2, dtype=np.uint64)
assert lib.bqr_llc_debug_stamps(buf.ctypes.data_as(ctypes.c_void_p), ctypes.c_size_t(buf.nbytes)) == 0
st = buf.reshape(W, 74, 2).astype(np.int64)
t0 = st[:, 70, 0].min()
rel = np.where(st > 0, st - t0, -1)
print("block0 start", rel[:, 70, 0].tolist(), "block1 start", rel[:, 71, 0].tolist(), "block1 left done", rel[:, 73, 0].tolist())
pub = rel[:, :66, 1].max(axis=0)       # publish time of v_k (by its owner)
got = np.where(rel[:, :66, 0] >= 0, rel[:, :66, 0], np.nan)
print(" k  publish(k)  min_wait_ret(k)  max_wait_ret(k)  step(k)=pub(k+1)-pub(k)")
for k in range(66):
    nxt = pub[k + 1] if k + 1 < 66 else -1
    print(f"{k:2d} {pub[k]:10d} {np.nanmin(got[:, k]):12.0f} {np.nanmax(got[:, k]):12.0f} {nxt - pub[k] if nxt > 0 and pub[k] > 0 else -1:10d}")
