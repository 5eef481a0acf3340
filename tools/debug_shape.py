"""Where does a shape's GPU factorisation differ from the oracle?
    python tools/debug_shape.py f32 128 128 [variant]"""
import os
import sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
if len(sys.argv) > 4:
    os.environ["BQR_FORCE_VARIANT"] = sys.argv[4]
import numpy as np  # noqa: E402
import bqr_inputs  # noqa: E402
import oracle  # noqa: E402
from oracle.compare import compare_geqrf  # noqa: E402
from gpu_util import geqrf_gpu  # noqa: E402
import paper_conf_ipps_andersonsk12_b200 as bqr  # noqa: E402

dt, m, n = sys.argv[1], int(sys.argv[2]), int(sys.argv[3])
batch = int(os.environ.get("DBG_BATCH", 4))
seed = int(os.environ.get("DBG_SEED", 3))
A = bqr_inputs.random_batch(m, n, batch, dt, seed=seed)
out, tau = geqrf_gpu(A, m)
rep = compare_geqrf(A, m, out, tau, full_q=m <= 200)
print(bqr.kernel_name(0 if dt == "f32" else 1, m, n), {k: rep[k] for k in rep if k != "fail_idx"})
ref, tref, _ = oracle.geqrf_cm(A, m)
fi = rep["fail_idx"][0] if rep["fail_idx"] else 0
print("failing matrices:", rep["fail_idx"])
R = np.triu(oracle.from_cm(out, m)[fi])
Rr = np.triu(oracle.from_cm(ref, m)[fi])
d = np.abs(np.abs(R) - np.abs(Rr))
bad = np.argwhere(d > 1e-3 * np.abs(Rr).max())
print("bad R entries:", len(bad), bad[:10].tolist())
print("tau diff first bad:", np.nonzero(np.abs(np.abs(tau[fi]) - np.abs(tref[fi])) > 1e-3)[0][:10])
