"""GPU parity of NEXT-3: bqr_getrf_np_batched (LU without
pivoting) and bqr_gauss_jordan_batched (Gauss-Jordan on [A | B]) through the
C ABI against the fp64 oracle (oracle.getrf_np_cm / gauss_jordan_cm, paper
Sec. III-A/B), on the paper's diagonally dominant inputs
(P:L1009), with the comparators of oracle/compare.py."""
import ctypes

import numpy as np
import pytest

import bqr_inputs
from oracle.compare import compare_gj, compare_lu

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a GPU", allow_module_level=True)

import paper_conf_ipps_andersonsk12_b200 as bqr  # noqa: E402


def _code(a):
    return bqr.R32 if a.dtype == np.float32 else bqr.C64


def lu_gpu(A_cm, m):
    batch, n, lda = A_cm.shape
    buf = torch.from_numpy(np.ascontiguousarray(A_cm)).cuda()
    info = torch.full((batch,), -7, dtype=torch.int32, device="cuda")
    st = bqr.load().bqr_getrf_np_batched(_code(A_cm), m, n, batch, ctypes.c_void_p(buf.data_ptr()), lda,
                                         ctypes.c_void_p(info.data_ptr()), None)
    assert st == 0, st
    torch.cuda.synchronize()
    return buf.cpu().numpy(), info.cpu().numpy()


def gj_gpu(A_cm, B_cm):
    batch, n, lda = A_cm.shape
    _, nrhs, ldb = B_cm.shape
    a = torch.from_numpy(np.ascontiguousarray(A_cm)).cuda()
    b = torch.from_numpy(np.ascontiguousarray(B_cm)).cuda()
    info = torch.full((batch,), -7, dtype=torch.int32, device="cuda")
    st = bqr.load().bqr_gauss_jordan_batched(_code(A_cm), n, nrhs, batch, ctypes.c_void_p(a.data_ptr()), lda,
                                             ctypes.c_void_p(b.data_ptr()), ldb, ctypes.c_void_p(info.data_ptr()),
                                             None)
    assert st == 0, st
    torch.cuda.synchronize()
    return a.cpu().numpy(), b.cpu().numpy(), info.cpu().numpy()


LU_SHAPES = [(1, 1), (2, 2), (3, 3), (7, 7), (8, 8), (9, 9), (16, 16), (17, 17), (31, 31), (32, 32), (33, 33),
             (56, 56), (63, 63), (64, 64), (65, 65), (100, 100), (127, 127), (128, 128)]


@pytest.mark.parametrize("m,n", LU_SHAPES)
@pytest.mark.parametrize("dt", ["f32", "c64"])
def test_lu_square(dt, m, n):
    A = bqr_inputs.diag_dominant_batch(n, 37, dt, seed=500 + n)
    out, info = lu_gpu(A, m)
    rep = compare_lu(A, m, out, info)
    assert rep["ok"], rep


@pytest.mark.parametrize("m,n", [(80, 16), (16, 80), (40, 100), (128, 9), (5, 3), (3, 5)])
@pytest.mark.parametrize("dt", ["f32", "c64"])
def test_lu_rectangular(dt, m, n):
    rng = np.random.default_rng(m * 1000 + n)
    A = bqr_inputs.random_batch(m, n, 21, dt, seed=600 + m + n)
    k = min(m, n)
    idx = np.arange(k)
    A[:, idx, idx] = (3.0 * max(m, n) * np.where(rng.random((21, k)) < 0.5, -1.0, 1.0)).astype(A.dtype)
    out, info = lu_gpu(A, m)
    rep = compare_lu(A, m, out, info)
    assert rep["ok"], rep


def test_lu_zero_pivot_info_exact():
    # exact integer matrices: a zero first pivot, a zero third pivot, a regular one
    mats = [np.array([[0, 1, 2], [1, 0, 1], [2, 1, 0]]),
            np.array([[1, 2, 3], [2, 4, 7], [3, 6, 1]]),   # u22 = 0 after step 1 -> info 2
            np.array([[4, 1, 0], [1, 4, 1], [0, 1, 4]])]
    A = np.stack([np.asarray(M, dtype=np.float32).T for M in mats])  # column-major storage
    out, info = lu_gpu(A, 3)
    assert list(info) == [1, 2, 0]
    rep = compare_lu(A, 3, out, info)
    assert rep["ok"], rep


def test_lu_lda_padding_untouched():
    n, lda = 40, 45
    A = bqr_inputs.diag_dominant_batch(n, 9, "f32", seed=9, lda=lda)
    out, info = lu_gpu(A, n)
    assert np.isnan(out[:, :, n:]).all()
    rep = compare_lu(A, n, out, info)
    assert rep["ok"], rep


@pytest.mark.parametrize("n,nrhs", [(1, 1), (2, 1), (4, 1), (7, 1), (8, 2), (15, 1), (16, 4), (31, 1), (32, 3),
                                    (56, 1), (63, 1), (64, 8), (100, 1), (120, 8), (127, 1)])
@pytest.mark.parametrize("dt", ["f32", "c64"])
def test_gauss_jordan(dt, n, nrhs):
    A = bqr_inputs.diag_dominant_batch(n, 29, dt, seed=700 + n)
    B = bqr_inputs.rhs_batch(n, nrhs, 29, dt, seed=800 + n)
    Ao, X, info = gj_gpu(A, B)
    rep = compare_gj(A, B, Ao, X, info)
    assert rep["ok"], rep


def test_gauss_jordan_zero_pivot_info_exact():
    mats = [np.array([[0, 1], [1, 0]]), np.array([[1, 2], [2, 4]]), np.array([[2, 1], [1, 3]])]
    A = np.stack([np.asarray(M, dtype=np.float32).T for M in mats])
    B = np.ones((3, 1, 2), dtype=np.float32)
    Ao, X, info = gj_gpu(A, B)
    assert list(info) == [1, 2, 0]
    np.testing.assert_allclose(X[2, 0], np.linalg.solve(mats[2], np.ones(2)), rtol=1e-6)


@pytest.mark.parametrize("name", ["L56", "GJ56"])
def test_bench_configs_full(name):
    """The bench's NEXT-3 workloads at full size (8,000 problems)."""
    cfg = bqr_inputs.CONFIGS[name]
    A = bqr_inputs.diag_dominant_batch(cfg["n"], cfg["batch"], cfg["dtype"], cfg["seed"])
    if name == "L56":
        out, info = lu_gpu(A, cfg["m"])
        rep = compare_lu(A, cfg["m"], out, info)
    else:
        B = bqr_inputs.rhs_batch(cfg["n"], cfg["nrhs"], cfg["batch"], cfg["dtype"], cfg["seed"])
        Ao, X, info = gj_gpu(A, B)
        rep = compare_gj(A, B, Ao, X, info)
    assert rep["ok"], rep


def test_lu_deterministic_and_slice_invariant():
    A = bqr_inputs.diag_dominant_batch(56, 300, "f32", seed=77)
    o1, _ = lu_gpu(A, 56)
    o2, _ = lu_gpu(A, 56)
    o3, _ = lu_gpu(A[123:124], 56)
    assert np.array_equal(o1, o2)
    assert np.array_equal(o1[123:124], o3)
