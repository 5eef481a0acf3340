import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np
import bqr_inputs, oracle
from oracle.compare import compare_geqrf
from gpu_util import geqrf_gpu
for dt in ["c64", "f32"]:
    for n in [4, 8, 16]:
        cases = bqr_inputs.edge_matrices(n, dt)
        for name, v in cases.items():
            A = oracle.to_cm(v[None])
            out, tau = geqrf_gpu(A, n)
            rep = compare_geqrf(A, n, out, tau)
            if not rep["ok"]:
                print(dt, n, name, {k: rep[k] for k in rep if k not in ("fail_idx",)})
                ref = oracle.geqrf_cm(A, n)
                print("gpu tau", tau, "\nref tau", ref[1])
                print("gpu out", out[0].T, "\nref", ref[0][0].T)
print("edge debug done")
