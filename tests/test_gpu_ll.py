"""GPU parity of the round-2 left-looking C3 class (csrc/bqr_ll.cuh,
`ll_f32_56x56_left4_x2`) on the paths the bench shape does not take: the
persistent warp loop (more pairs than one resident round), odd batches (the
spare half-warp), even lda > m (row-pair loads into padded storage), and the
fallbacks to the right-looking class (odd lda, 4-byte-aligned base).
Comparator: oracle/compare.py (north-star tolerances, reading Q10)."""
import ctypes

import numpy as np
import pytest

import bqr_inputs
from oracle.compare import compare_geqrf

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a GPU", allow_module_level=True)

import paper_conf_ipps_andersonsk12_b200 as bqr  # noqa: E402
from gpu_util import geqrf_gpu  # noqa: E402


def test_dispatch_is_left_looking():
    assert bqr.kernel_name(bqr.R32, 56, 56) == "ll_f32_56x56_left4_x2"


def test_persistent_loop_second_pass():
    """5,100 matrices = 2,550 pairs on <= 148 CTAs of 17 warps: chunk 18, so
    warp 0 of every CTA factors a second pair (matrices 36 b + 34, 36 b + 35)
    after its first; those and a sample of the rest against the oracle."""
    batch = 5100
    A = bqr_inputs.random_batch(56, 56, batch, "f32", seed=5100)
    out, tau = geqrf_gpu(A, 56)
    second = [i for b in range(0, 148, 5) for i in (36 * b + 34, 36 * b + 35) if i < batch]
    idx = sorted(set(second) | set(range(0, batch, 97)) | {batch - 1})
    rep = compare_geqrf(A[idx], 56, out[idx], tau[idx])
    assert rep["ok"], rep


@pytest.mark.parametrize("batch", [1, 2, 3, 33, 149, 297])
def test_odd_and_small_batches(batch):
    A = bqr_inputs.random_batch(56, 56, batch, "f32", seed=700 + batch)
    out, tau = geqrf_gpu(A, 56)
    rep = compare_geqrf(A, 56, out, tau)
    assert rep["ok"], rep


@pytest.mark.parametrize("lda", [58, 64, 57])
def test_lda_padding(lda):
    """even lda: the left-looking class (8-byte row-pair accesses); odd lda:
    the right-looking class of the same shape.  NaN sentinels in the padding
    rows must survive untouched."""
    A = bqr_inputs.random_batch(56, 56, 71, "f32", seed=lda, lda=lda)
    out, tau = geqrf_gpu(A, 56)
    rep = compare_geqrf(A, 56, out, tau)
    assert rep["ok"] and rep["padding_ok"], rep


def test_four_byte_aligned_base():
    """A base that is 4- but not 8-byte aligned takes the right-looking class."""
    batch = 40
    A = bqr_inputs.random_batch(56, 56, batch, "f32", seed=77)
    flat = torch.zeros(A.size + 1, dtype=torch.float32, device="cuda")
    flat[1:] = torch.from_numpy(np.ascontiguousarray(A).reshape(-1)).cuda()
    tau = torch.empty((batch, 56), dtype=torch.float32, device="cuda")
    st = bqr.load().bqr_geqrf_batched(bqr.R32, 56, 56, batch, ctypes.c_void_p(flat.data_ptr() + 4), 56,
                                      ctypes.c_void_p(tau.data_ptr()),
                                      ctypes.c_void_p(torch.cuda.current_stream().cuda_stream))
    assert st == 0
    torch.cuda.synchronize()
    out = flat[1:].cpu().numpy().reshape(A.shape)
    rep = compare_geqrf(A, 56, out, tau.cpu().numpy())
    assert rep["ok"], rep


# ------------------------------------------------------------ left-looking LU (bqr_lll.cuh)
def _lu_gpu(A_cm, m):
    batch, n, lda = A_cm.shape
    buf = torch.from_numpy(np.ascontiguousarray(A_cm)).cuda()
    info = torch.full((batch,), -7, dtype=torch.int32, device="cuda")
    st = bqr.load().bqr_getrf_np_batched(bqr.R32, m, n, batch, ctypes.c_void_p(buf.data_ptr()), lda,
                                         ctypes.c_void_p(info.data_ptr()), None)
    assert st == 0, st
    torch.cuda.synchronize()
    return buf.cpu().numpy(), info.cpu().numpy()


def test_lu56_zero_pivot_info():
    """Row 30 zero left of and on the diagonal: l_30,j = 0 for j < 30, so
    u_30,30 = a_30,30 = 0 exactly -> scale 0, info = 31, the elimination goes
    on (reading L1); matrix 0 also has a zero first pivot (info 1)."""
    from oracle.compare import compare_lu
    A = bqr_inputs.diag_dominant_batch(56, 5, "f32", seed=56)  # storage (batch, col, row)
    A[1, :31, 30] = 0.0
    A[0, 0, :] = 0.0
    out, info = _lu_gpu(A, 56)
    assert list(info[:2]) == [1, 31] and list(info[2:]) == [0, 0, 0]
    rep = compare_lu(A, 56, out, info)
    assert rep["ok"], rep


@pytest.mark.parametrize("lda", [58, 57])
def test_lu56_lda_padding(lda):
    from oracle.compare import compare_lu
    A = bqr_inputs.diag_dominant_batch(56, 35, "f32", seed=lda, lda=lda)
    out, info = _lu_gpu(A, 56)
    assert np.isnan(out[:, :, 56:]).all()
    rep = compare_lu(A, 56, out, info)
    assert rep["ok"], rep


@pytest.mark.parametrize("batch", [1, 3, 10067])
def test_lu56_batches(batch):
    """odd batches (spare half-warp) and a batch whose CTAs factor up to
    three pairs per warp (persistent loop), sampled against the oracle"""
    from oracle.compare import compare_lu
    A = bqr_inputs.diag_dominant_batch(56, batch, "f32", seed=900 + batch)
    out, info = _lu_gpu(A, 56)
    idx = sorted(set(range(0, batch, 53)) | {batch - 1})
    rep = compare_lu(A[idx], 56, out[idx], info[idx])
    assert rep["ok"], rep


# ------------------------------------------------------------ left-looking Gauss-Jordan (bqr_llgj.cuh)
def _gj_gpu(A_cm, B_cm):
    batch, n, lda = A_cm.shape
    _, nrhs, ldb = B_cm.shape
    a = torch.from_numpy(np.ascontiguousarray(A_cm)).cuda()
    b = torch.from_numpy(np.ascontiguousarray(B_cm)).cuda()
    info = torch.full((batch,), -7, dtype=torch.int32, device="cuda")
    st = bqr.load().bqr_gauss_jordan_batched(bqr.R32, n, nrhs, batch, ctypes.c_void_p(a.data_ptr()), lda,
                                             ctypes.c_void_p(b.data_ptr()), ldb, ctypes.c_void_p(info.data_ptr()),
                                             None)
    assert st == 0, st
    torch.cuda.synchronize()
    return a.cpu().numpy(), b.cpu().numpy(), info.cpu().numpy()


def test_gj56_dispatch():
    assert bqr.load().bqr_lu_kernel_name(bqr.R32, 56, 56, 1, 1).decode() == "llgj_f32_56x57_left4_x2"


@pytest.mark.parametrize("batch", [1, 3, 37, 10067])
def test_gj56_batches(batch):
    from oracle.compare import compare_gj
    A = bqr_inputs.diag_dominant_batch(56, batch, "f32", seed=1200 + batch)
    B = bqr_inputs.rhs_batch(56, 1, batch, "f32", seed=1300 + batch)
    Ao, X, info = _gj_gpu(A, B)
    idx = sorted(set(range(0, batch, 53)) | {batch - 1})
    rep = compare_gj(A[idx], B[idx], Ao[idx], X[idx], info[idx])
    assert rep["ok"], rep


def test_gj56_zero_pivot_info():
    """row 30 zero left of and on the diagonal: pivot 30 is exactly zero after
    the eliminations (scale 0, info 31, the elimination goes on, reading L1);
    matrix 0 has a zero first pivot (info 1)"""
    from oracle.compare import compare_gj
    A = bqr_inputs.diag_dominant_batch(56, 4, "f32", seed=561)
    B = bqr_inputs.rhs_batch(56, 1, 4, "f32", seed=562)
    A[1, :31, 30] = 0.0
    A[0, 0, :] = 0.0
    Ao, X, info = _gj_gpu(A, B)
    assert list(info[:2]) == [1, 31] and list(info[2:]) == [0, 0]
    rep = compare_gj(A, B, Ao, X, info)
    assert rep["ok"], rep


@pytest.mark.parametrize("lda,ldb", [(58, 60), (57, 56), (56, 57)])
def test_gj56_leading_dims(lda, ldb):
    """even lda / ldb: the left-looking class; an odd one: lu_rf_kernel"""
    from oracle.compare import compare_gj
    A = bqr_inputs.diag_dominant_batch(56, 21, "f32", seed=lda + ldb, lda=lda)
    B = bqr_inputs.rhs_batch(56, 1, 21, "f32", seed=ldb, ldb=ldb) if "ldb" in bqr_inputs.rhs_batch.__code__.co_varnames \
        else np.pad(bqr_inputs.rhs_batch(56, 1, 21, "f32", seed=ldb), ((0, 0), (0, 0), (0, ldb - 56)),
                    constant_values=np.nan)
    Ao, X, info = _gj_gpu(A, B)
    rep = compare_gj(A, B, Ao, X, info)
    assert rep["ok"], rep
