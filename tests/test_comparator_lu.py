"""Self-tests of the NEXT-3 comparators (oracle.compare.compare_lu /
compare_gj): single-precision LAPACK results (scipy sgetrf on column
dominant inputs, where it does not pivot; numpy ssolve) pass; perturbed L,
U, X, a wrong info and an unscaled column fail."""
import numpy as np
import scipy.linalg

import bqr_inputs
import oracle
from oracle.compare import compare_gj, compare_lu


def _lapack_lu_cm(A_cm, n):
    out = np.empty_like(A_cm)
    for b in range(A_cm.shape[0]):
        A = A_cm[b].T[:n, :]
        P, L, U = scipy.linalg.lu(A)
        assert np.array_equal(P, np.eye(n))
        out[b] = (np.tril(L, -1) + np.triu(U)).astype(A_cm.dtype).T
    return out


def test_lu_comparator_accepts_fp32_lapack_and_rejects_errors():
    for dt in ("f32", "c64"):
        A_cm = bqr_inputs.diag_dominant_batch(56, 6, dt, 3)
        info = np.zeros(6, dtype=np.int32)
        lu = _lapack_lu_cm(A_cm, 56)
        assert compare_lu(A_cm, 56, lu, info)["ok"]
        bad = lu.copy()
        bad[2, 10, 30] *= 1.01  # an L entry (storage [b, col, row]: row 30 > col 10)
        assert not compare_lu(A_cm, 56, bad, info)["ok"]
        bad = lu.copy()
        bad[1, 40, 5] += 0.01 * np.abs(lu[1]).max()  # a U entry (row 5 < col 40)
        assert not compare_lu(A_cm, 56, bad, info)["ok"]
        bad = lu.copy()
        bad[0, 3, 4:] /= lu[0, 3, 3]  # column 3 scaled twice
        assert not compare_lu(A_cm, 56, bad, info)["ok"]
        wrong_info = info.copy()
        wrong_info[4] = 7
        assert not compare_lu(A_cm, 56, lu, wrong_info)["ok"]


def test_gj_comparator_accepts_fp32_solve_and_rejects_errors():
    for dt in ("f32", "c64"):
        A_cm = bqr_inputs.diag_dominant_batch(32, 5, dt, 4)
        B_cm = bqr_inputs.rhs_batch(32, 2, 5, dt, 4)
        A = np.swapaxes(A_cm, 1, 2)
        B = np.swapaxes(B_cm, 1, 2)
        X = np.linalg.solve(A, B).astype(A_cm.dtype)
        X_cm = np.ascontiguousarray(np.swapaxes(X, 1, 2))
        Aref_cm, _, _ = oracle.gauss_jordan_cm(A_cm, B_cm)
        A_out = Aref_cm.astype(A_cm.dtype)
        info = np.zeros(5, dtype=np.int32)
        assert compare_gj(A_cm, B_cm, A_out, X_cm, info)["ok"]
        bad = X_cm.copy()
        bad[3, 1, 7] *= 1.001
        assert not compare_gj(A_cm, B_cm, A_out, bad, info)["ok"]
        bad_a = A_out.copy()
        bad_a[2, 5, 9] += 0.01 * np.abs(A_cm[2]).max()
        assert not compare_gj(A_cm, B_cm, bad_a, X_cm, info)["ok"]
        assert not compare_gj(A_cm, B_cm, A_out, X_cm, np.ones(5, dtype=np.int32))["ok"]
