"""Pins for the oracle's least-squares solve (oracle.gels, paper Sec. III-D,
P:L309-317: factor A, apply Q^T to b "appended to the right side of the
matrix", then "solve the upper triangular system using row operations").

Pinned against things other than the oracle itself:
  * hand-worked closed forms (tests/golden/gels_examples.json): a line fit,
    a square integer system, a complex 2x1 projection;
  * LAPACK: scipy.linalg.lstsq (xGELSD, an SVD-based solver: a different
    algorithm) on random full-rank systems;
  * invariants: normal equations A^H (A x - b) = 0, ||A x - b|| equal to the
    norm of the returned residual components, square consistent systems
    solved exactly, rank deficiency reported through info.
A wrong conjugate, a skipped row operation, a transposed R or a missing
Q^H apply fails at least one of them.
"""
import json
import os

import numpy as np
import pytest
import scipy.linalg

import oracle

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "gels_examples.json")


def _c(x):
    a = np.array(x, dtype=np.float64)
    return a[..., 0] + 1j * a[..., 1]


def _cases():
    with open(GOLDEN) as f:
        return json.load(f)["cases"]


@pytest.mark.parametrize("case", _cases(), ids=lambda c: c["name"])
def test_gels_worked_examples(case):
    cplx = case["dtype"] == "c128"
    conv = _c if cplx else (lambda x: np.array(x, dtype=np.float64))
    A, b, x_exp = conv(case["A"]), conv(case["b"]), conv(case["x"])
    X, res, info = oracle.gels(A, b)
    assert info[0] == 0
    np.testing.assert_allclose(X[0], x_exp, rtol=0, atol=1e-14)
    np.testing.assert_allclose(np.linalg.norm(res[0]), case["residual_norm"], rtol=1e-14, atol=1e-15)


@pytest.mark.parametrize("shape", [(3, 2), (8, 8), (56, 56), (240, 66), (80, 16), (192, 96), (17, 5)])
@pytest.mark.parametrize("cplx", [False, True])
@pytest.mark.parametrize("nrhs", [1, 3])
def test_gels_vs_lapack_lstsq(shape, cplx, nrhs):
    m, n = shape
    rng = np.random.default_rng(m * 1000 + n + 7 * nrhs + cplx)
    A = rng.standard_normal((2, m, n))
    B = rng.standard_normal((2, m, nrhs))
    if cplx:
        A = A + 1j * rng.standard_normal((2, m, n))
        B = B + 1j * rng.standard_normal((2, m, nrhs))
    X, res, info = oracle.gels(A, B)
    assert (info == 0).all()
    for b in range(2):
        x_ref, rss, rank, sv = scipy.linalg.lstsq(A[b], B[b])
        assert rank == n
        kappa = sv[0] / sv[-1]
        scale = np.abs(x_ref).max()
        np.testing.assert_allclose(X[b], x_ref, rtol=0, atol=1e-13 * kappa ** 2 * max(scale, 1.0))
        # residual components carry the residual norm (xGELS convention)
        r = A[b] @ X[b] - B[b]
        np.testing.assert_allclose(np.linalg.norm(res[b], axis=0), np.linalg.norm(r, axis=0), rtol=1e-10,
                                   atol=1e-13 * kappa * np.linalg.norm(B[b]))


@pytest.mark.parametrize("cplx", [False, True])
def test_gels_normal_equations(cplx):
    rng = np.random.default_rng(11)
    m, n = 240, 66
    A = rng.standard_normal((m, n)) + (1j * rng.standard_normal((m, n)) if cplx else 0)
    b = rng.standard_normal((m, 1)) + (1j * rng.standard_normal((m, 1)) if cplx else 0)
    X, _, _ = oracle.gels(A, b)
    g = A.conj().T @ (A @ X[0] - b)  # gradient of ||Ax-b||^2 / 2: zero at the minimiser
    assert np.abs(g).max() <= 1e-11 * np.linalg.norm(A) * (np.linalg.norm(A) * np.linalg.norm(X[0]) + np.linalg.norm(b))


def test_gels_square_exact_and_consistent():
    # a consistent tall system: b = A x* exactly -> x*, zero residual
    rng = np.random.default_rng(5)
    A = rng.integers(-4, 5, size=(9, 4)).astype(np.float64)
    xs = rng.integers(-3, 4, size=(4, 2)).astype(np.float64)
    X, res, info = oracle.gels(A, A @ xs)
    assert info[0] == 0
    np.testing.assert_allclose(X[0], xs, atol=1e-12)
    assert np.abs(res[0]).max() <= 1e-12


def test_gels_rank_deficient_info():
    # a zero column: R_11 == 0 exactly -> info = 2 (1-based), as LAPACK xTRTRS
    A = np.array([[1.0, 0.0, 2.0], [2.0, 0.0, 1.0], [2.0, 0.0, 3.0], [1.0, 0.0, 1.0]])
    b = np.ones((4, 1))
    _, _, info = oracle.gels(A, b)
    assert info[0] == 2


def test_gels_agrees_with_geqrf_plus_apply():
    # the LS path is geqrf -> Q^H B -> back substitution: its R and Q^H b are
    # exactly the standalone factorisation's (same oracle arithmetic)
    rng = np.random.default_rng(3)
    A = rng.standard_normal((3, 20, 7))
    B = rng.standard_normal((3, 20, 2))
    Ao, tau, Bo, _ = oracle.gels_cm(oracle.to_cm(A), 20, oracle.to_cm(B))
    RV, tau2, _ = oracle.geqrf(A)
    np.testing.assert_array_equal(oracle.from_cm(Ao, 20), RV)
    np.testing.assert_array_equal(tau, tau2)
    QhB = oracle.apply_qh(RV, tau2, B)
    np.testing.assert_array_equal(oracle.from_cm(Bo, 20)[:, 7:, :], QhB[:, 7:, :])
    R = np.triu(RV[:, :7, :])
    X = oracle.from_cm(Bo, 20)[:, :7, :]
    np.testing.assert_allclose(np.einsum("bij,bjk->bik", R, X), QhB[:, :7, :], atol=1e-13)
