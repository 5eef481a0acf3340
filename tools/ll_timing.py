"""Phase timeline of the left-looking C3 kernel (debug build with
-DBQR_LL_TIMING): per warp of CTA 0, cycles from the CTA's first stamp to
each block's start / end of its left-looking applies / end of its panels.

    python tools/ll_timing.py abl/libbqr_lltime.so
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
W, E = 17, 13
w = bench.Workload("C3", 0, 1, torch, bqr, batch=int(sys.argv[2]) if len(sys.argv) > 2 else None)
for _ in range(3):
    w.restore()
    torch.cuda.synchronize()
    w.geqrf()
    torch.cuda.synchronize()
buf = np.zeros(W * E, dtype=np.uint64)
assert lib.bqr_ll_debug_stamps(buf.ctypes.data_as(ctypes.c_void_p), ctypes.c_size_t(buf.nbytes)) == 0
st = buf.reshape(W, E).astype(np.int64)
st = st[st[:, 0] > 0]
W = st.shape[0]
t0 = st[:, 0].min()
rel = st - t0
print("warp " + " ".join(f"{n:>7s}" for n in ["b0", "b0L", "b0P", "b1", "b1L", "b1P", "b2", "b2L", "b2P", "b3", "b3L", "b3P", "end"]))
for i in range(W):
    print(f"{i:4d} " + " ".join(f"{x:7d}" for x in rel[i]))
d = np.diff(rel, axis=1)
names = ["b0 left", "b0 panels", "b0->b1", "b1 left", "b1 panels", "b1->b2", "b2 left", "b2 panels", "b2->b3", "b3 left",
         "b3 panels", "tail"]
print("mean phase cycles: " + ", ".join(f"{n}={m:.0f}" for n, m in zip(names, d.mean(axis=0))))
