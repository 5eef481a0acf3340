"""One bqr_geqrf_wy_batched call on the C5 c64 cell n (the command ncu wraps)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bqr_inputs  # noqa: E402
import paper_conf_ipps_andersonsk12_b200 as bqr  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 256
cfg = bqr_inputs.c5_config(n, "c64")
B = cfg["batch"]
buf = torch.from_numpy(bqr_inputs.random_batch(n, n, B, "c64", cfg["seed"])).cuda()
tau = torch.empty((B, n), dtype=buf.dtype, device="cuda")
wsb = bqr.geqrf_wy_workspace_bytes(bqr.C64, n, n, n, B)
ws = torch.empty(wsb, dtype=torch.uint8, device="cuda")
for _ in range(int(sys.argv[2]) if len(sys.argv) > 2 else 1):
    st = bqr.geqrf_wy_batched_ptr(bqr.C64, n, n, B, buf.data_ptr(), n, tau.data_ptr(), ws.data_ptr(), wsb)
    assert st == 0
torch.cuda.synchronize()
print("done")
