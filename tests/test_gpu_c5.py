"""C5 (BASELINE.json config 5: square size sweep, fp32 and complex64; the
paper's Fig. 9 / Fig. 11 sweeps) at the bench's per-GPU
batch sizes and launch configuration (bqr_inputs.c5_config, bench.py
C5_CELLS): the whole batch is factored in one call and every 97th matrix
plus the last is compared with the fp64 oracle."""
import numpy as np
import pytest

import bqr_inputs
from oracle.compare import compare_geqrf

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a GPU", allow_module_level=True)

import paper_conf_ipps_andersonsk12_b200 as bqr  # noqa: E402

CELLS = [(16, "f32"), (56, "f32"), (128, "f32"), (256, "f32"), (16, "c64"), (56, "c64"), (128, "c64"),
         (256, "c64")]


@pytest.mark.parametrize("n,dt", CELLS, ids=[f"{d}_{n}" for n, d in CELLS])
def test_c5_cell_full_batch_sampled(n, dt):
    n_sm = torch.cuda.get_device_properties(0).multi_processor_count
    cfg = bqr_inputs.c5_config(n, dt, n_sm=n_sm)
    A = bqr_inputs.random_batch(n, n, cfg["batch"], dt, cfg["seed"], cfg["dist"])
    buf = torch.from_numpy(A).cuda()
    tau = torch.empty((cfg["batch"], n), dtype=buf.dtype, device="cuda")
    code = bqr.R32 if dt == "f32" else bqr.C64
    st = bqr.geqrf_batched_ptr(code, n, n, cfg["batch"], buf.data_ptr(), n, tau.data_ptr(),
                               torch.cuda.current_stream().cuda_stream)
    assert st == 0
    torch.cuda.synchronize()
    idx = np.array(sorted(set(range(0, cfg["batch"], 97)) | {cfg["batch"] - 1}))
    ti = torch.from_numpy(idx).cuda()
    out = buf.index_select(0, ti).cpu().numpy()
    tu = tau.index_select(0, ti).cpu().numpy()
    rep = compare_geqrf(A[idx], n, out, tu, full_q=n <= 128)
    assert rep["ok"], rep
