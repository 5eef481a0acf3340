"""A few geqrf launches of B random 240 x 66 complex64 matrices through
whatever class the dispatch (or BQR_FORCE_VARIANT) picks -- the command ncu
wraps for the cluster-per-matrix captures.

    BQR_FORCE_VARIANT=alt_cl2_c64_256x72_aug python tools/cl_once.py 32
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_andersonsk12_b200 as bqr  # noqa: E402

b = int(sys.argv[1]) if len(sys.argv) > 1 else 32
A0 = torch.randn(b, 66, 240, dtype=torch.complex64, device="cuda")
A = torch.empty_like(A0)
tau = torch.empty(b, 66, dtype=torch.complex64, device="cuda")
for _ in range(3):
    A.copy_(A0)
    assert bqr.geqrf_batched_ptr(bqr.C64, 240, 66, b, A.data_ptr(), 240, tau.data_ptr(),
                                 torch.cuda.current_stream().cuda_stream) == 0
torch.cuda.synchronize()
print("done", bqr.kernel_name(bqr.C64, 240, 66))
