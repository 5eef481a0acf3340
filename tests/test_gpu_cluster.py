"""GPU parity of the cluster-per-matrix complex classes (csrc/bqr_cl.cuh:
`alt_cl4_c64_256x72[_aug]`, `alt_cl2_c64_256x72[_aug]`,
`alt_cl1_c64_256x72_aug`; one cluster of 4 / 2 / 1 CTAs per matrix,
reflectors pushed to every CTA by st.async into distributed shared memory,
or by shared stores + mbarrier arrives on one CTA).  They are explicit variants (BQR_FORCE_VARIANT, read once per
process), so each runs in a child process that compares geqrf and the fused
Q^H B against the fp64 oracle (oracle/compare.py, north-star tolerances) and
prints one JSON line.  Shapes: the STAP shape, the class bound 256 x 72,
ragged row/column counts, 1 x 1 / 2 x 2 / 256 x 1 matrices (the complex
1-row reflector), a batch larger than the resident clusters
(the persistent loop and its ring-phase continuation), several right-hand
sides."""
import json
import os
import subprocess
import sys

import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a GPU", allow_module_level=True)

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r"""
import sys, json
sys.path.insert(0, ROOT); sys.path.insert(0, ROOT + '/tests')
import paper_conf_ipps_andersonsk12_b200 as bqr
import bqr_inputs
from oracle.compare import compare_geqrf, compare_apply
from gpu_util import geqrf_gpu, geqrf_qhb_gpu
lib = bqr.load()
res = {'kernel': bqr.kernel_name(bqr.C64, 240, 66), 'qhb_kernel': lib.bqr_qhb_kernel_name(bqr.C64, 240, 66, 1).decode(),
       'resident': lib.bqr_resident_matrices(bqr.C64, 240, 66), 'cases': []}
for m, n, b, seed in ((240, 66, 7, 11), (256, 72, 5, 12), (255, 71, 3, 13), (131, 40, 4, 14), (33, 33, 3, 15),
                      (240, 66, 2 * res['resident'] + 5, 16), (1, 1, 3, 17), (2, 2, 3, 18), (256, 1, 3, 19),
                      (72, 72, 2, 20)):
    A = bqr_inputs.random_batch(m, n, b, 'c64', seed=seed)
    out, tau = geqrf_gpu(A, m)
    idx = sorted(set(range(0, b, max(1, b // 12))) | {b - 1})
    rep = compare_geqrf(A[idx], m, out[idx], tau[idx], full_q=False)
    res['cases'].append({'op': 'geqrf', 'shape': [m, n, b], 'ok': bool(rep['ok'])})
for m, n, nrhs, b, seed in ((240, 66, 1, 9, 21), (240, 66, 6, 5, 22), (200, 60, 3, 4, 23)):
    A = bqr_inputs.random_batch(m, n, b, 'c64', seed=seed)
    B = bqr_inputs.rhs_batch(m, nrhs, b, 'c64', seed=seed)
    out, tau, QhB = geqrf_qhb_gpu(A, m, B)
    r1 = compare_geqrf(A, m, out, tau, full_q=False)
    r2 = compare_apply(out, m, min(m, n), tau, B, QhB)
    res['cases'].append({'op': 'qhb', 'shape': [m, n, nrhs, b], 'ok': bool(r1['ok'] and r2['ok'])})
print(json.dumps(res))
"""


@pytest.mark.parametrize("variant", ["alt_cl4_c64_256x72_aug", "alt_cl2_c64_256x72_aug", "alt_cl1_c64_256x72_aug"])
def test_cluster_class_parity(variant):
    env = dict(os.environ, BQR_FORCE_VARIANT=variant)
    out = subprocess.run([sys.executable, "-c", f"ROOT = {ROOT!r}\n" + CHILD], env=env, capture_output=True,
                         text=True, timeout=600)
    assert out.returncode == 0, out.stderr[-3000:]
    res = json.loads(out.stdout.strip().splitlines()[-1])
    assert res["kernel"] == variant and res["qhb_kernel"] == variant, res
    assert res["resident"] > 0, res
    bad = [c for c in res["cases"] if not c["ok"]]
    assert not bad, bad
