"""GPU parity of the compact-WY blocked variant (bqr_geqrf_wy_batched,
bqr_wy.cu): register-file panels of 96 columns + tensor-core trailing
updates C - V (T^H (V^H C)), against the fp64 oracle with the north-star
tolerances (reading Q10), for the complex shapes beyond one SM (C5's
192 / 224 / 256 and ragged ones), chunked workspaces, bitwise determinism
and the forwarding of shapes without a blocked variant."""
import numpy as np
import pytest

import bqr_inputs
from oracle.compare import compare_geqrf

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a GPU", allow_module_level=True)

import paper_conf_ipps_andersonsk12_b200 as bqr  # noqa: E402


def wy_gpu(A_cm, m, chunk=None):
    batch, n, lda = A_cm.shape
    buf = torch.from_numpy(np.ascontiguousarray(A_cm)).cuda()
    tau = torch.full((batch, min(m, n)), float("nan"), dtype=buf.dtype, device="cuda")
    chunk = batch if chunk is None else chunk
    code = bqr.C64 if np.iscomplexobj(A_cm) else bqr.R32
    wsb = max(1, bqr.geqrf_wy_workspace_bytes(code, m, n, lda, chunk))
    ws = torch.empty(wsb, dtype=torch.uint8, device="cuda")
    st = bqr.geqrf_wy_batched_ptr(code, m, n, batch, buf.data_ptr(), lda, tau.data_ptr(), ws.data_ptr(), wsb)
    assert st == 0, bqr.load().bqr_status_string(st)
    torch.cuda.synchronize()
    return buf.cpu().numpy(), tau.cpu().numpy()


@pytest.mark.parametrize("m,n", [(192, 192), (224, 224), (256, 256), (256, 200), (176, 176), (256, 161),
                                 (240, 180), (128, 128), (160, 160), (98, 97)])
def test_wy_parity(m, n):
    assert "tcgen05" in bqr.load().bqr_geqrf_wy_kernel_name(bqr.C64, m, n, m).decode()
    A = bqr_inputs.random_batch(m, n, 24, "c64", seed=5000 + m + n)
    out, tau = wy_gpu(A, m)
    rep = compare_geqrf(A, m, out, tau, full_q=False)
    assert rep["ok"], rep
    assert rep["residual_max"] < 3e-6 and rep["orth_max"] < 5e-6, rep


@pytest.mark.parametrize("m,n", [(256, 256), (192, 192), (224, 224), (128, 128), (96, 96), (256, 100), (200, 65)])
def test_wy_parity_f32(m, n):
    """fp32: 64-column register panels + real FastF32 tensor-core GEMMs."""
    assert "wy_f32_panel64" in bqr.load().bqr_geqrf_wy_kernel_name(bqr.R32, m, n, m).decode()
    A = bqr_inputs.random_batch(m, n, 24, "f32", seed=6000 + m + n)
    out, tau = wy_gpu(A, m)
    rep = compare_geqrf(A, m, out, tau, full_q=m <= 128)
    assert rep["ok"], rep


def test_wy_chunked_and_deterministic():
    """A workspace for 5 matrices processes 23 in 5 chunks; results are
    bitwise equal to the one-chunk run and across runs."""
    A = bqr_inputs.random_batch(256, 256, 23, "c64", seed=71)
    o1, t1 = wy_gpu(A, 256)
    o2, t2 = wy_gpu(A, 256, chunk=5)
    o3, t3 = wy_gpu(A, 256, chunk=5)
    assert np.array_equal(o1.view(np.uint32), o2.view(np.uint32)) and np.array_equal(t1.view(np.uint32), t2.view(np.uint32))
    assert np.array_equal(o2.view(np.uint32), o3.view(np.uint32))
    assert compare_geqrf(A, 256, o1, t1, full_q=False)["ok"]


def test_wy_forwards_unsupported_shapes():
    """Shapes without a blocked variant (one panel wide, or rows that are not
    a 16-byte multiple) take bqr_geqrf_batched."""
    for m, n, dt in ((64, 64, "c64"), (99, 97, "c64"), (130, 130, "f32")):
        A = bqr_inputs.random_batch(m, n, 8, dt, seed=72)
        out, tau = wy_gpu(A, m)
        assert compare_geqrf(A, m, out, tau, full_q=False)["ok"]
        code = bqr.C64 if dt == "c64" else bqr.R32
        assert bqr.load().bqr_geqrf_wy_kernel_name(code, m, n, m).decode() == bqr.kernel_name(code, m, n)


@pytest.mark.parametrize("dt", ["c64", "f32"])
@pytest.mark.parametrize("kind", ["graded", "near_rank", "tiny", "huge"])
def test_wy_contract_edges(kind, dt):
    A = bqr_inputs.stress_batch(256, 256, 6, dt, kind, seed=73)
    out, tau = wy_gpu(A, 256)
    rep = compare_geqrf(A, 256, out, tau, full_q=False)
    assert rep["ok"], {k: v for k, v in rep.items() if k != "fail_idx"}
