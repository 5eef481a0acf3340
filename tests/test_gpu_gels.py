"""GPU parity of the least-squares path bqr_gels_batched (paper Sec. III-D,
P:L309-317; STAP weight solve, Sec. VII) against the oracle's fp64 QR solve,
through the C ABI, with oracle.compare.compare_gels (backward error 1e-6,
condition-scaled forward error 1e-5, residual components 1e-4)."""
import numpy as np
import pytest

import bqr_inputs
import oracle
from oracle.compare import compare_gels, compare_geqrf

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a GPU", allow_module_level=True)

from gpu_util import gels_gpu  # noqa: E402


def _problem(m, n, nrhs, dtype, batch, seed, lda=None, ldb=None):
    A = bqr_inputs.random_batch(m, n, batch, dtype, seed, "normal", lda=lda)
    B = bqr_inputs.random_batch(m, nrhs, batch, dtype, seed + 1, "normal", lda=ldb)
    return A, B


def _check(A, m, B):
    Ao, tau, Bo, info = gels_gpu(A, m, B)
    rep = compare_gels(A, m, B, Bo, info)
    assert rep["ok"], rep
    # the factorisation left in A is the geqrf one
    rg = compare_geqrf(A, m, Ao, tau, full_q=m <= 128)
    assert rg["ok"], rg
    return Ao, Bo, info, rep


def test_stap_240x66_full_batch():
    """C4's STAP shape with its right-hand side: 256 complex 240x66 solves."""
    A = bqr_inputs.config_batch("C4")
    B = bqr_inputs.rhs_batch(240, 1, 256, "c64", seed=4)
    _check(A, 240, B)


@pytest.mark.parametrize("m,n,nrhs,dt", [
    (8, 8, 1, "f32"), (56, 56, 1, "f32"), (56, 40, 3, "f32"), (100, 37, 2, "f32"), (128, 128, 1, "f32"),
    (256, 64, 1, "f32"), (33, 33, 1, "f32"), (200, 150, 1, "f32"), (256, 256, 1, "f32"),
    (80, 16, 1, "c64"), (192, 96, 1, "c64"), (64, 64, 2, "c64"), (240, 66, 4, "c64"), (17, 5, 1, "c64"),
    (160, 160, 1, "c64"), (256, 240, 1, "c64"), (4, 4, 1, "f32"), (1, 1, 1, "f32"), (5, 1, 2, "c64"),
])
def test_gels_shapes(m, n, nrhs, dt):
    A, B = _problem(m, n, nrhs, dt, batch=37, seed=m * 7 + n + nrhs)
    _check(A, m, B)


def test_gels_padding_and_strides():
    """lda > m and ldb > m: NaN sentinels in the padding rows stay untouched."""
    A, B = _problem(50, 20, 2, "f32", batch=9, seed=3, lda=53, ldb=57)
    Ao, Bo, _, _ = _check(A, 50, B)
    assert np.isnan(Ao[:, :, 50:]).all() and np.isnan(Bo[:, :, 50:]).all()


def test_gels_zero_column_reports_info():
    """A zero column gives R_jj == 0 exactly: info = j+1 (LAPACK xTRTRS), the
    rest of the batch is solved normally."""
    A, B = _problem(30, 6, 1, "f32", batch=5, seed=9)
    A[2, 3, :] = 0.0  # matrix 2, column 3
    Ao, tau, Bo, info = gels_gpu(A, 30, B)
    assert list(info) == [0, 0, 4, 0, 0]
    rep = compare_gels(A, 30, B, Bo, info)
    assert rep["ok"], rep


def test_gels_consistent_system_exact():
    """b = A x* with small integers: the solve recovers x* to fp32 accuracy
    and the residual components vanish."""
    rng = np.random.default_rng(4)
    A = rng.integers(-3, 4, size=(16, 40, 12)).astype(np.float32)
    xs = rng.integers(-2, 3, size=(16, 12, 1)).astype(np.float32)
    b = np.einsum("bij,bjk->bik", A.astype(np.float64), xs.astype(np.float64)).astype(np.float32)
    A_cm, B_cm = oracle.to_cm(A), oracle.to_cm(b)
    _, _, Bo, info = gels_gpu(A_cm, 40, B_cm)
    assert (info == 0).all()
    X = oracle.from_cm(Bo, 40)
    np.testing.assert_allclose(X[:, :12], xs, atol=2e-4)
    assert np.abs(X[:, 12:]).max() < 1e-4


def test_gels_deterministic():
    A, B = _problem(240, 66, 1, "c64", batch=20, seed=12)
    r1 = gels_gpu(A, 240, B)
    r2 = gels_gpu(A, 240, B)
    for x, y in zip(r1, r2):
        assert np.array_equal(x.view(np.uint8), y.view(np.uint8))
