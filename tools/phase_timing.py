"""Per-step phase timing of the first matrix of CTA 0 (debug build with
-DBQR_PHASE_TIMING, headline classes).  Prints, per step, the CTA-wide step
duration (max over warps of end - min entry) and the mean per-warp phase
durations: wait, slotP/reflector, apply-rest.

    python tools/phase_timing.py C4 abl/libbqr_dbg.so
"""
import ctypes
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_ipps_andersonsk12_b200 as bqr  # noqa: E402

cfg = sys.argv[1]
bqr._LIB_PATH = os.path.abspath(sys.argv[2])
lib = bqr.load()
S, W = 300, 32
w = bench.Workload(cfg, 0, 1, torch, bqr, batch=int(sys.argv[3]) if len(sys.argv) > 3 else None)
for it in range(3):
    w.restore()
    lib.bqr_debug_clear()
    torch.cuda.synchronize()
    w.geqrf()
    torch.cuda.synchronize()
buf = np.zeros(S * W * 4, dtype=np.uint64)
assert lib.bqr_debug_stamps(buf.ctypes.data_as(ctypes.c_void_p), ctypes.c_size_t(buf.nbytes)) == 0
st = buf.reshape(S, W, 4).astype(np.int64)
used = st[:, :, 0] != 0
nsteps = int(used.any(axis=1).sum())
warps = np.where(used.any(axis=0))[0]
t0 = st[0, warps, 0][st[0, warps, 0] > 0].min()
rows = []
for k in range(nsteps):
    e = st[k, warps, :]
    ok = e[:, 0] > 0
    e = e[ok]
    ent, wt, mid, end = e[:, 0] - t0, e[:, 1] - t0, e[:, 2] - t0, e[:, 3] - t0
    midv = np.where(e[:, 2] > 0, mid, wt)
    rows.append(dict(k=k, entry_min=int(ent.min()), end_max=int(end.max()),
                     wait=float(np.mean(wt - ent)), slotp=float(np.mean(midv - wt)), rest=float(np.mean(end - midv)),
                     step=int(end.max() - ent.min())))
# owner analysis (CTA classes with one column group per warp, G = warps):
# the owner of column k+1 stamps phase 2 right after publishing v_{k+1}
G = len(warps)
prev_pub = None
for k, r in enumerate(rows):
    w = (k + 1) % G
    if k + 1 < nsteps and st[k, w, 2] > 0:
        pub = st[k, w, 2] - t0
        r["own_chain"] = int(st[k, w, 2] - st[k, w, 1])  # v_k received -> v_{k+1} published
        r["period"] = int(pub - prev_pub) if prev_pub is not None else None
        prev_pub = pub
for r in rows:
    print(json.dumps(r))
tot = rows[-1]["end_max"] - rows[0]["entry_min"]
print(json.dumps({"total_cycles": int(tot), "steps": nsteps, "warps": len(warps),
                  "mean_wait": float(np.mean([r["wait"] for r in rows])),
                  "mean_slotp": float(np.mean([r["slotp"] for r in rows])),
                  "mean_rest": float(np.mean([r["rest"] for r in rows]))}))
