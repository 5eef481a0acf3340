"""Pins for the oracle (oracle/bqr_ref.c) against things other than itself:
hand-worked closed forms (tests/golden/worked_examples.json), LAPACK
(scipy d/zgeqrf, d/zorgqr, d/zormqr -- the paper's 'consistent with LAPACK',
P:L305), invariants that hold for any Householder QR, and brute-force Givens
rotations on tiny inputs.  Chosen so that a dropped term, a wrong sign, a
missing conjugate or a transposed operand in the oracle fails at least one.
"""
import json
import os

import numpy as np
import pytest
import scipy.linalg
import scipy.linalg.lapack as lapack

import oracle

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "worked_examples.json")


def _parse(x, cplx):
    a = np.array(x, dtype=object)
    if cplx:
        a = np.array(x, dtype=np.float64)
        return a[..., 0] + 1j * a[..., 1]
    return np.array([[float(v) for v in row] for row in x], dtype=np.float64) if a.ndim == 2 else np.array([float(v) for v in x])


def _cases():
    with open(GOLDEN) as f:
        return json.load(f)["cases"]


@pytest.mark.parametrize("case", _cases(), ids=lambda c: c["name"])
def test_worked_examples(case):
    cplx = case["dtype"] == "c128"
    A = _parse(case["A"], cplx)
    RV_exp = _parse(case["RV"], cplx)
    tau_exp = np.array(case["tau"], dtype=np.float64)
    if cplx:
        tau_exp = tau_exp[..., 0] + 1j * tau_exp[..., 1]
    RV, tau, margin = oracle.geqrf(A[None])
    np.testing.assert_allclose(RV[0], RV_exp, rtol=1e-13, atol=1e-14)
    np.testing.assert_allclose(tau[0], tau_exp, rtol=1e-13, atol=1e-14)
    # the sign-tie margin |alpha|/nu the comparator's flip rule relies on
    np.testing.assert_allclose(margin[0], np.array(case["margin"]), rtol=1e-13, atol=1e-15)


def test_minus_zero_sign_rule():
    """Q4: alpha = -0.0 flips beta's sign (copysign), +0.0 does not."""
    Ap = np.array([[[0.0, 1.0], [1.0, 1.0]]])
    Am = np.array([[[-0.0, 1.0], [1.0, 1.0]]])
    assert oracle.geqrf(Ap)[0][0, 0, 0] == -1.0
    assert oracle.geqrf(Am)[0][0, 0, 0] == 1.0


def _scipy_geqrf(A):
    f = lapack.zgeqrf if np.iscomplexobj(A) else lapack.dgeqrf
    qr, tau, work, info = f(A)
    assert info == 0
    return qr, tau


SHAPES = [(1, 1), (2, 1), (1, 3), (3, 3), (5, 5), (8, 8), (7, 3), (3, 7), (16, 9), (20, 20), (33, 17), (56, 56), (64, 66), (240, 66)]


@pytest.mark.parametrize("cplx", [False, True])
@pytest.mark.parametrize("shape", SHAPES)
def test_vs_lapack_geqrf(shape, cplx):
    """Library special case: the oracle IS LAPACK xGEQR2 (blocked xGEQRF gives
    the same factors up to rounding), so V, tau and R agree to ~1e-12."""
    m, n = shape
    rng = np.random.default_rng(m * 1000 + n + (7 if cplx else 0))
    A = rng.standard_normal((m, n))
    if cplx:
        A = A + 1j * rng.standard_normal((m, n))
    RV, tau, _ = oracle.geqrf(A[None])
    qr, tau_l = _scipy_geqrf(A.copy())
    scale = np.abs(A).max()
    np.testing.assert_allclose(RV[0], qr, rtol=0, atol=1e-12 * scale * max(m, n))
    np.testing.assert_allclose(tau[0], tau_l, rtol=0, atol=1e-12 * max(m, n))


@pytest.mark.parametrize("cplx", [False, True])
@pytest.mark.parametrize("shape", [(4, 4, 4), (9, 5, 5), (12, 7, 4), (30, 30, 30), (240, 66, 66)])
def test_vs_lapack_orgqr(shape, cplx):
    m, n, k = shape
    rng = np.random.default_rng(m + 31 * n + k)
    A = rng.standard_normal((m, n)) + (1j * rng.standard_normal((m, n)) if cplx else 0)
    qr, tau = _scipy_geqrf(A.copy())
    f = lapack.zungqr if cplx else lapack.dorgqr
    q_l, work, info = f(qr[:, :n].copy(), tau[:k].copy())
    assert info == 0
    # LAPACK orgqr with k < n uses only the first k reflectors
    Q = oracle.orgqr(qr[None, :, :n], tau[None, :k], n)
    np.testing.assert_allclose(Q[0], q_l, rtol=0, atol=1e-12 * m)


@pytest.mark.parametrize("cplx", [False, True])
@pytest.mark.parametrize("shape", [(4, 4, 1), (8, 8, 3), (240, 66, 1), (80, 16, 2), (10, 3, 5)])
def test_vs_lapack_apply_qh(shape, cplx):
    m, n, nrhs = shape
    rng = np.random.default_rng(3 * m + n + nrhs)
    A = rng.standard_normal((m, n)) + (1j * rng.standard_normal((m, n)) if cplx else 0)
    B = rng.standard_normal((m, nrhs)) + (1j * rng.standard_normal((m, nrhs)) if cplx else 0)
    qr, tau = _scipy_geqrf(A.copy())
    if cplx:
        lwork = lapack.zunmqr("L", "C", qr, tau, B.copy(), -1)[1][0].real
        C, work, info = lapack.zunmqr("L", "C", qr, tau, B.copy(), int(lwork))
    else:
        lwork = lapack.dormqr("L", "T", qr, tau, B.copy(), -1)[1][0]
        C, work, info = lapack.dormqr("L", "T", qr, tau, B.copy(), int(lwork))
    assert info == 0
    got = oracle.apply_qh(qr[None], tau[None], B[None])
    np.testing.assert_allclose(got[0], C, rtol=0, atol=1e-12 * m)


# ---------------------------------------------------------------- invariants

@pytest.mark.parametrize("cplx", [False, True])
@pytest.mark.parametrize("shape", [(6, 6), (40, 25), (56, 56), (240, 66)])
def test_invariants(shape, cplx):
    m, n = shape
    rng = np.random.default_rng(17 + m + n)
    A = rng.standard_normal((3, m, n)) + (1j * rng.standard_normal((3, m, n)) if cplx else 0)
    RV, tau, margin = oracle.geqrf(A)
    R = np.triu(RV)[:, :n, :]
    # column norms preserved: ||R e_j|| = ||A e_j|| (H orthogonal)
    np.testing.assert_allclose(np.linalg.norm(R, axis=1), np.linalg.norm(A, axis=1), rtol=1e-12)
    # R = D chol(A^H A)^H with D = diag(+-1)
    for b in range(3):
        L = np.linalg.cholesky(np.conj(A[b].T) @ A[b])
        d = np.sign(np.real(np.diag(R[b])))
        np.testing.assert_allclose(d[:, None] * R[b], np.conj(L.T), rtol=0, atol=1e-10 * np.abs(A[b]).max() * m)
    # diagonal of R is real
    assert np.all(np.imag(np.diagonal(R, axis1=1, axis2=2)) == 0)
    # tau ranges: real in [1,2]; complex |1 - tau| <= 1 and Re tau in [1,2]
    t = tau
    nz = t != 0
    assert np.all((np.real(t[nz]) >= 1 - 1e-14) & (np.real(t[nz]) <= 2 + 1e-14))
    if cplx:
        assert np.all(np.abs(1 - t) <= 1 + 1e-14)
    else:
        assert np.all(np.imag(t) == 0)
    # orthogonality and reconstruction in double
    Q = oracle.orgqr(RV, tau, m)
    np.testing.assert_allclose(np.conj(np.swapaxes(Q, 1, 2)) @ Q, np.broadcast_to(np.eye(m), (3, m, m)), atol=1e-13 * m)
    np.testing.assert_allclose(Q[:, :, :n] @ R, A, atol=1e-13 * m * np.abs(A).max())
    assert np.all((margin >= 0) & (margin <= 1))


def test_det_preserved():
    rng = np.random.default_rng(5)
    A = rng.standard_normal((4, 12, 12))
    RV, tau, _ = oracle.geqrf(A)
    detR = np.prod(np.diagonal(RV, axis1=1, axis2=2), axis=1)
    np.testing.assert_allclose(np.abs(detR), np.abs(np.linalg.det(A)), rtol=1e-11)


def test_upper_triangular_input_untouched():
    rng = np.random.default_rng(6)
    A = np.triu(rng.standard_normal((2, 9, 9)))
    RV, tau, _ = oracle.geqrf(A)
    assert np.all(tau == 0)
    np.testing.assert_array_equal(RV, A)


@pytest.mark.parametrize("cplx", [False, True])
def test_augmented_least_squares(cplx):
    """append b to A; (Q^H b)[0:n] appears in column n and
    |R_aug[n,n]| is the least-squares residual min ||Ax - b||."""
    rng = np.random.default_rng(9)
    m, n = 30, 8
    A = rng.standard_normal((m, n)) + (1j * rng.standard_normal((m, n)) if cplx else 0)
    b = rng.standard_normal((m, 1)) + (1j * rng.standard_normal((m, 1)) if cplx else 0)
    RVa, taua, _ = oracle.geqrf(np.concatenate([A, b], axis=1)[None])
    RV, tau, _ = oracle.geqrf(A[None])
    qhb = oracle.apply_qh(RV, tau, b[None])[0]
    np.testing.assert_allclose(RVa[0, :n, n], qhb[:n, 0], atol=1e-12)
    x, res, *_ = np.linalg.lstsq(A, b, rcond=None)
    np.testing.assert_allclose(abs(RVa[0, n, n]), np.sqrt(res[0]), rtol=1e-10)
    # solve R x = (Q^H b)[0:n] by back substitution (scipy) == lstsq
    xs = scipy.linalg.solve_triangular(np.triu(RV[0, :n, :n]), qhb[:n])
    np.testing.assert_allclose(xs, x, atol=1e-10)


# ---------------------------------------------------------------- brute force

def _givens_r(A):
    """Textbook Givens QR (real): zero below-diagonal entries bottom-up."""
    R = A.astype(np.float64).copy()
    m, n = R.shape
    for j in range(min(m, n)):
        for i in range(m - 1, j, -1):
            a, b = R[i - 1, j], R[i, j]
            if b == 0:
                continue
            r = np.hypot(a, b)
            c, s = a / r, b / r
            G = np.array([[c, s], [-s, c]])
            R[[i - 1, i], :] = G @ R[[i - 1, i], :]
    return np.triu(R)


def _mgs_r(A):
    """Modified Gram-Schmidt (complex-capable): R with positive diagonal."""
    A = A.astype(np.complex128).copy()
    m, n = A.shape
    R = np.zeros((n, n), dtype=np.complex128)
    for j in range(n):
        R[j, j] = np.linalg.norm(A[:, j])
        q = A[:, j] / R[j, j]
        for l in range(j + 1, n):
            R[j, l] = np.vdot(q, A[:, l])
            A[:, l] -= R[j, l] * q
    return R


@pytest.mark.parametrize("seed", range(6))
def test_bruteforce_givens(seed):
    rng = np.random.default_rng(100 + seed)
    m = 2 + seed % 5
    n = 1 + (seed * 3) % m
    A = rng.standard_normal((m, n)) + np.eye(m, n) * 3  # well conditioned
    RV, _, _ = oracle.geqrf(A[None])
    Rg = _givens_r(A)
    np.testing.assert_allclose(np.abs(np.triu(RV[0])), np.abs(Rg), atol=1e-12)


@pytest.mark.parametrize("seed", range(4))
def test_bruteforce_mgs_complex(seed):
    """|R| row-wise equals Gram-Schmidt's up to a unimodular row phase; LAPACK
    keeps the diagonal real, so the phase is +-1."""
    rng = np.random.default_rng(200 + seed)
    m, n = 6, 4
    A = rng.standard_normal((m, n)) + 1j * rng.standard_normal((m, n)) + 2 * np.eye(m, n)
    RV, _, _ = oracle.geqrf(A[None])
    R = np.triu(RV[0])[:n]
    Rm = _mgs_r(A)
    d = np.sign(np.real(np.diag(R)))
    np.testing.assert_allclose(d[:, None] * R, Rm, atol=1e-12)


def test_batch_and_lda_layout():
    """Batch stride lda*n, padding rows untouched, batch position invariant."""
    rng = np.random.default_rng(11)
    m, n, lda, batch = 5, 4, 7, 6
    A_cm = rng.standard_normal((batch, n, lda))
    A_cm[:, :, m:] = np.nan
    out, tau, _ = oracle.geqrf_cm(A_cm, m)
    assert np.all(np.isnan(out[:, :, m:]))
    for b in range(batch):
        single, t1, _ = oracle.geqrf_cm(A_cm[b:b + 1], m)
        np.testing.assert_array_equal(single[0, :, :m], out[b, :, :m])
        np.testing.assert_array_equal(t1[0], tau[b])


def test_threads_do_not_change_bits():
    rng = np.random.default_rng(12)
    A = rng.standard_normal((64, 20, 20))
    oracle.set_threads(1)
    a1 = oracle.geqrf(A)[0]
    oracle.set_threads(0)
    a2 = oracle.geqrf(A)[0]
    np.testing.assert_array_equal(a1, a2)
