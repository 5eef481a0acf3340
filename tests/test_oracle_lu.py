"""Pins for the oracle's NEXT-3 factorisations (oracle.getrf_np,
oracle.gauss_jordan; paper Sec. III-A/B, Listings 5-7).

Pinned against things other than the oracle itself:
  * hand-worked closed forms (tests/golden/lu_gj_examples.json), including
    the zero-pivot "notsolved" flag of Listing 5 and a complex system;
  * LAPACK special case: scipy.linalg.lu (xGETRF, partial pivoting) on
    column diagonally dominant matrices, where partial pivoting provably
    makes no row interchange, so P = I and L, U must agree;
  * library solves: numpy.linalg.solve (xGESV) for Gauss-Jordan, and an
    LU-based forward/back substitution (scipy solve_triangular) -- a
    different algorithm reaching the same x;
  * invariants: L U = A, det A = prod(diag U), upper-triangular input
    unchanged; brute force: Cramer's rule on 3x3 systems.
A dropped Schur-complement term, a transposed multiplier, a row scaled by
the pivot instead of its reciprocal's product, or an update that skips the
rows above the pivot in Gauss-Jordan fails at least one of them.
"""
import json
import os

import numpy as np
import pytest
import scipy.linalg

import bqr_inputs
import oracle

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "lu_gj_examples.json")


def _conv(x, cplx):
    a = np.array(x, dtype=np.float64)
    return a[..., 0] + 1j * a[..., 1] if cplx else a


def _cases():
    with open(GOLDEN) as f:
        return json.load(f)["cases"]


@pytest.mark.parametrize("case", _cases(), ids=lambda c: c["name"])
def test_worked_examples(case):
    cplx = case["dtype"] == "c128"
    A = _conv(case["A"], cplx)
    LU, info = oracle.getrf_np(A)
    assert info[0] == case["info"]
    np.testing.assert_allclose(LU[0], _conv(case["lu"], cplx), rtol=0, atol=1e-15)
    if "b" in case:
        b = _conv(case["b"], cplx)[:, None]
        X, info = oracle.gauss_jordan(A, b)
        assert info[0] == 0
        np.testing.assert_allclose(X[0, :, 0], _conv(case["x"], cplx), rtol=0, atol=1e-15)
    if "gj_a_exit" in case:
        n = A.shape[0]
        Aout, _, _ = oracle.gauss_jordan_cm(oracle.to_cm(A[None]), oracle.to_cm(_conv(case["b"], cplx)[None, :, None]))
        np.testing.assert_allclose(oracle.from_cm(Aout, n)[0], _conv(case["gj_a_exit"], cplx), rtol=0, atol=1e-15)


def test_gauss_jordan_zero_pivot_flag():
    X, info = oracle.gauss_jordan(np.array([[0.0, 1.0], [1.0, 0.0]]), np.array([[1.0], [2.0]]))
    assert info[0] == 1
    X, info = oracle.gauss_jordan(np.array([[1.0, 2.0], [2.0, 4.0]]), np.array([[1.0], [2.0]]))
    assert info[0] == 2


def _dd(n, batch, cplx, seed):
    A_cm = bqr_inputs.diag_dominant_batch(n, batch, "c64" if cplx else "f32", seed)
    return oracle.from_cm(A_cm, n).astype(np.complex128 if cplx else np.float64)


@pytest.mark.parametrize("n", [1, 2, 5, 16, 56, 96])
@pytest.mark.parametrize("cplx", [False, True])
def test_lu_matches_lapack_getrf_without_interchanges(n, cplx):
    A = _dd(n, 4, cplx, 10 + n)
    LU, info = oracle.getrf_np(A)
    assert (info == 0).all()
    for b in range(A.shape[0]):
        P, L, U = scipy.linalg.lu(A[b])
        np.testing.assert_array_equal(P, np.eye(n))  # column dominance: no interchange
        np.testing.assert_allclose(np.tril(LU[b], -1) + np.eye(n), L, rtol=1e-12, atol=1e-13)
        np.testing.assert_allclose(np.triu(LU[b]), U, rtol=1e-12, atol=1e-12 * np.abs(U).max())


@pytest.mark.parametrize("m,n", [(6, 6), (9, 4), (4, 9), (56, 56), (80, 16)])
@pytest.mark.parametrize("cplx", [False, True])
def test_lu_reconstructs_a(m, n, cplx):
    rng = np.random.default_rng(m * 100 + n)
    A = rng.standard_normal((3, m, n)) + (1j * rng.standard_normal((3, m, n)) if cplx else 0)
    k = min(m, n)
    for j in range(k):  # dominant leading diagonal so no pivot is tiny
        A[:, j, j] += 3 * max(m, n) * (1 if j % 2 == 0 else -1)
    LU, info = oracle.getrf_np(A)
    assert (info == 0).all()
    L = np.tril(LU, -1)[:, :, :k] + np.eye(m, k)
    U = np.triu(LU)[:, :k, :]
    np.testing.assert_allclose(L @ U, A, rtol=0, atol=1e-12 * np.abs(A).max())


@pytest.mark.parametrize("n", [3, 8, 56])
def test_det_is_product_of_pivots(n):
    A = _dd(n, 3, False, 7)
    LU, _ = oracle.getrf_np(A)
    d = np.prod(np.diagonal(LU, axis1=1, axis2=2), axis=1)
    np.testing.assert_allclose(d, np.linalg.det(A), rtol=1e-10)


def test_upper_triangular_input_unchanged():
    rng = np.random.default_rng(3)
    U = np.triu(rng.standard_normal((7, 7))) + 5 * np.eye(7)
    LU, info = oracle.getrf_np(U)
    assert info[0] == 0
    np.testing.assert_array_equal(LU[0], U)


@pytest.mark.parametrize("n,nrhs", [(1, 1), (4, 1), (16, 3), (56, 1), (96, 2)])
@pytest.mark.parametrize("cplx", [False, True])
def test_gauss_jordan_matches_lapack_solve(n, nrhs, cplx):
    A = _dd(n, 3, cplx, 40 + n)
    rng = np.random.default_rng(n)
    B = rng.standard_normal((3, n, nrhs)) + (1j * rng.standard_normal((3, n, nrhs)) if cplx else 0)
    X, info = oracle.gauss_jordan(A, B)
    assert (info == 0).all()
    np.testing.assert_allclose(X, np.linalg.solve(A, B), rtol=1e-11, atol=1e-12)
    # a different algorithm: LU (no pivoting) + forward/back substitution
    LU, _ = oracle.getrf_np(A)
    for b in range(3):
        y = scipy.linalg.solve_triangular(LU[b], B[b], lower=True, unit_diagonal=True)
        x = scipy.linalg.solve_triangular(LU[b], y, lower=False)
        np.testing.assert_allclose(X[b], x, rtol=1e-11, atol=1e-12)


def test_gauss_jordan_cramer_brute_force():
    rng = np.random.default_rng(11)
    for _ in range(20):
        A = rng.standard_normal((3, 3)) + 4 * np.eye(3)
        b = rng.standard_normal(3)
        det = np.linalg.det(A)
        cramer = []
        for j in range(3):
            Aj = A.copy()
            Aj[:, j] = b
            cramer.append(np.linalg.det(Aj) / det)
        X, info = oracle.gauss_jordan(A, b[:, None])
        np.testing.assert_allclose(X[0, :, 0], cramer, rtol=1e-12, atol=1e-13)


def test_diag_dominant_inputs_are_dominant():
    A = _dd(24, 5, True, 1)
    mag = np.abs(A)
    d = np.diagonal(mag, axis1=1, axis2=2)
    assert (d > mag.sum(axis=1) - d).all() and (d > mag.sum(axis=2) - d).all()
