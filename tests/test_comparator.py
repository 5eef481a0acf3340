"""The parity comparator (oracle/compare.py) accepts an independent correct
fp32 factorisation (scipy LAPACK sgeqrf/cgeqrf) and rejects plausible bugs."""
import numpy as np
import pytest
import scipy.linalg.lapack as lapack

import bqr_inputs
import oracle
from oracle.compare import compare_geqrf, compare_apply, compare_orgqr


def _lapack32(A_cm, m):
    """Factor each matrix with single-precision LAPACK; returns (out_cm, tau)."""
    batch, n, lda = A_cm.shape
    out = A_cm.copy()
    taus = []
    f = lapack.cgeqrf if np.iscomplexobj(A_cm) else lapack.sgeqrf
    for b in range(batch):
        qr, tau, _, info = f(np.asfortranarray(A_cm[b, :, :m].T))
        assert info == 0
        out[b, :, :m] = qr.T
        taus.append(tau)
    return out, np.array(taus)


@pytest.mark.parametrize("m,n,dt", [(8, 8, "f32"), (56, 56, "f32"), (240, 66, "c64"), (33, 20, "c64")])
def test_accepts_lapack_fp32(m, n, dt):
    A = bqr_inputs.random_batch(m, n, 20, dt, seed=5)
    out, tau = _lapack32(A, m)
    rep = compare_geqrf(A, m, out, tau)
    assert rep["ok"], rep
    assert rep["residual_max"] < 1e-6 and rep["orth_max"] < 5e-6


def test_rejects_perturbed_r():
    A = bqr_inputs.random_batch(16, 16, 8, "f32", seed=6)
    out, tau = _lapack32(A, 16)
    out[3, 10, 2] *= 1.001  # R[2,10]
    rep = compare_geqrf(A, 16, out, tau)
    assert not rep["ok"] and 3 in rep["fail_idx"]


def test_rejects_wrong_tau():
    A = bqr_inputs.random_batch(16, 16, 8, "f32", seed=7)
    out, tau = _lapack32(A, 16)
    tau = tau.copy()
    tau[5, 4] *= 1.01
    rep = compare_geqrf(A, 16, out, tau)
    assert not rep["ok"] and 5 in rep["fail_idx"]


def test_rejects_unconjugated_update():
    """A complex factorisation whose trailing update used tau instead of
    conj(tau) (reading Q9) must fail."""
    rng = np.random.default_rng(8)
    m = n = 6
    A = (rng.standard_normal((m, n)) + 1j * rng.standard_normal((m, n))).astype(np.complex128)
    R = A.copy()
    taus = []
    for i in range(n):
        alpha = R[i, i]
        x = R[i + 1:, i]
        nu = np.sqrt(abs(alpha) ** 2 + np.vdot(x, x).real)
        beta = -np.copysign(nu, alpha.real)
        tau = complex((beta - alpha.real) / beta, -alpha.imag / beta)
        v = np.concatenate([[1.0], x / (alpha - beta)])
        R[i + 1:, i] = v[1:]
        R[i, i] = beta
        C = R[i:, i + 1:]
        C -= tau * np.outer(v, np.conj(v) @ C)  # BUG: should be conj(tau)
        taus.append(tau)
    A_cm = oracle.to_cm(A[None].astype(np.complex64))
    out_cm = oracle.to_cm(R[None].astype(np.complex64))
    rep = compare_geqrf(A_cm, m, out_cm, np.array([taus]))
    assert not rep["ok"]


def test_rejects_unjustified_sign_flip():
    """Flip the sign of row 0 of R and of reflector 0's Householder sign: a
    valid QR, but LAPACK's sign rule fixes it when |alpha|/nu is large."""
    A = bqr_inputs.random_batch(5, 5, 1, "f32", seed=9)
    out, tau = _lapack32(A, 5)
    logical = np.swapaxes(out, 1, 2).copy()
    logical[0, 0, :] *= -1  # R row 0 negated: A = (Q D)(D R) still holds only if Q changes too
    out2 = np.swapaxes(logical, 1, 2).copy()
    rep = compare_geqrf(A, 5, out2, tau)
    assert not rep["ok"]


def test_zero_matrix_exact():
    A = np.zeros((2, 4, 4), np.float32)
    out = A.copy()
    tau = np.zeros((2, 4), np.float32)
    assert compare_geqrf(A, 4, out, tau)["ok"]
    tau[1, 0] = 1e-30
    assert not compare_geqrf(A, 4, out, tau)["ok"]


def test_apply_and_orgqr_comparators():
    A = bqr_inputs.random_batch(12, 5, 4, "c64", seed=10)
    out, tau = _lapack32(A, 12)
    B = bqr_inputs.rhs_batch(12, 2, 4, "c64", seed=10)
    ref = oracle.apply_qh_cm(out.astype(np.complex128), 12, 5, tau, B)
    assert compare_apply(out, 12, 5, tau, B, ref.astype(np.complex64))["ok"]
    bad = ref.copy()
    bad[1, 0, 3] += 1e-3
    assert not compare_apply(out, 12, 5, tau, B, bad)["ok"]
    Q = oracle.orgqr_cm(out.astype(np.complex128), 12, 5, tau)
    assert compare_orgqr(out, 12, 5, tau, Q.astype(np.complex64))["ok"]
    Q[0, 1, 1] += 1e-3
    assert not compare_orgqr(out, 12, 5, tau, Q)["ok"]


def test_accepts_cascade_after_tie_flip():
    """A factorisation that takes the other sign at a near-tie pivot (column
    0, alpha ~ 0) legitimately differs in later pivot signs: accepted."""
    rng = np.random.default_rng(21)
    m = n = 8
    A = rng.standard_normal((m, n))
    A[0, 0] = 1e-9  # |alpha| / nu ~ 1e-9: the sign rule is a coin toss here
    R = A.copy()
    taus = []
    for i in range(n):
        alpha, x = R[i, i], R[i + 1:, i]
        nu = np.sqrt(alpha ** 2 + x @ x)
        beta = np.copysign(nu, alpha) if i == 0 else -np.copysign(nu, alpha)  # other sign at the tie
        tau = (beta - alpha) / beta if x.size else 0.0
        v = np.concatenate([[1.0], x / (alpha - beta)]) if x.size else np.array([1.0])
        if x.size:
            R[i + 1:, i] = v[1:]
            R[i, i] = beta
            C = R[i:, i + 1:]
            C -= tau * np.outer(v, v @ C)
        taus.append(tau)
    A_cm = oracle.to_cm(A[None].astype(np.float32))
    out_cm = oracle.to_cm(R[None].astype(np.float32))
    rep = compare_geqrf(A_cm, m, out_cm, np.array([taus], dtype=np.float32))
    assert rep["flips"] >= 1 and rep["ok"], rep


# ---------------------------------------------------------------- gels
def _ls_problem(m, n, cplx, seed=0, batch=3):
    rng = np.random.default_rng(seed)
    A = rng.standard_normal((batch, m, n))
    B = rng.standard_normal((batch, m, 1))
    if cplx:
        A = A + 1j * rng.standard_normal((batch, m, n))
        B = B + 1j * rng.standard_normal((batch, m, 1))
    dt = np.complex64 if cplx else np.float32
    return oracle.to_cm(A.astype(dt)), oracle.to_cm(B.astype(dt))


@pytest.mark.parametrize("m,n,cplx", [(240, 66, True), (56, 56, False), (80, 16, True)])
def test_compare_gels_accepts_fp32_lapack(m, n, cplx):
    """Single-precision LAPACK xGELS output passes the comparator."""
    import scipy.linalg.lapack as L
    from oracle.compare import compare_gels
    A_cm, B_cm = _ls_problem(m, n, cplx)
    Bout = B_cm.copy()
    fn = L.cgels if cplx else L.sgels
    for b in range(A_cm.shape[0]):
        A = oracle.from_cm(A_cm[b:b + 1], m)[0]
        bb = oracle.from_cm(B_cm[b:b + 1], m)[0]
        res = fn(A.copy(), bb.copy())
        Bout[b] = oracle.to_cm(res[1][None])[0]
    rep = compare_gels(A_cm, m, B_cm, Bout, np.zeros(A_cm.shape[0], np.int32))
    assert rep["ok"], rep


def test_compare_gels_rejects_wrong_solutions():
    from oracle.compare import compare_gels
    A_cm, B_cm = _ls_problem(240, 66, True)
    _, _, Bo, info = oracle.gels_cm(A_cm, 240, B_cm)
    good = Bo.astype(np.complex64)
    assert compare_gels(A_cm, 240, B_cm, good, info)["ok"]
    bad = good.copy()
    bad[0, 0, 5] *= 1.001  # one solution entry off by 1e-3 relative
    assert not compare_gels(A_cm, 240, B_cm, bad, info)["ok"]
    conj = good.copy()
    conj[:, :, :66] = np.conj(conj[:, :, :66])  # a dropped conjugate
    assert not compare_gels(A_cm, 240, B_cm, conj, info)["ok"]
    assert not compare_gels(A_cm, 240, B_cm, good, info + 1)["ok"]  # wrong info


def _householder_sign_rule(A, flip):
    """Unblocked Householder QR (xGEQR2 form: [R; V], tau) in fp64 with the
    LAPACK sign rule beta = -copysign(nu, Re alpha) or, flip=True,
    the opposite sign beta = +copysign(nu, Re alpha) (a self-consistent QR,
    i.e. A = Q R exactly, that is NOT LAPACK's)."""
    m, n = A.shape
    R = A.astype(np.complex128 if np.iscomplexobj(A) else np.float64).copy()
    taus = []
    for i in range(min(m, n)):
        alpha = R[i, i]
        x = R[i + 1:, i]
        nu = np.sqrt(abs(alpha) ** 2 + np.vdot(x, x).real)
        beta = np.copysign(nu, np.real(alpha)) * (1.0 if flip else -1.0)
        tau = (beta - alpha) / beta
        v = np.concatenate([[1.0], x / (alpha - beta)])
        R[i + 1:, i] = v[1:]
        R[i, i] = beta
        C = R[i:, i + 1:]
        C -= np.conj(tau) * np.outer(v, np.conj(v) @ C)
        taus.append(tau)
    return R, np.array(taus)


@pytest.mark.parametrize("cplx", [False, True])
def test_rejects_wrong_sign_rule_consistent_qr(cplx):
    """Every beta sign flipped, V and tau consistent with it: the residual and
    orthogonality checks pass (it IS a QR of A), so only the comparator's
    flip rule (oracle margin = |Re alpha|/nu well above 1e-4) can reject it.
    Pins the margin output of the oracle and the bad-flip rule together: with
    the margin forced to 0 (every flip 'allowed') this QR would be accepted."""
    rng = np.random.default_rng(31 + cplx)
    m, n, batch = 12, 9, 6
    outs, taus, As = [], [], []
    for _ in range(batch):
        A = rng.standard_normal((m, n))
        if cplx:
            A = A + 1j * rng.standard_normal((m, n))
        R, t = _householder_sign_rule(A, flip=True)
        As.append(A)
        outs.append(R)
        taus.append(t)
    dt = np.complex64 if cplx else np.float32
    A_cm = oracle.to_cm(np.array(As).astype(dt))
    out_cm = oracle.to_cm(np.array(outs).astype(dt))
    rep = compare_geqrf(A_cm, m, out_cm, np.array(taus).astype(dt))
    assert rep["residual_max"] < 1e-5 and rep["orth_max"] < 1e-5, rep
    assert rep["bad_flips"] > 0 and not rep["ok"], rep
    # the rejection comes from the oracle's margins: zeroed, a complex QR
    # would pass (real ones are also caught by the tau range [1, 2])
    ref_cm, tau_ref, margin = oracle.geqrf_cm(A_cm, m, with_margin=True)
    rep0 = compare_geqrf(A_cm, m, out_cm, np.array(taus).astype(dt), ref=(ref_cm, tau_ref, np.zeros_like(margin)))
    assert rep0["bad_flips"] == 0
    assert rep0["ok"] if cplx else not rep0["invariants_ok"], rep0
    # control: the same construction with LAPACK's sign rule is accepted
    outs = [_householder_sign_rule(A, flip=False) for A in As]
    rep = compare_geqrf(A_cm, m, oracle.to_cm(np.array([o[0] for o in outs]).astype(dt)),
                        np.array([o[1] for o in outs]).astype(dt))
    assert rep["ok"] and rep["bad_flips"] == 0, rep


def test_flip_rule_honours_ties():
    """A flip at an exact tie (margin 0, alpha = +0) is allowed; the same
    flip where the margin is large is not (bad_flips counts it)."""
    A = np.array([[0.0, 1.0, 2.0], [1.0, 1.0, 0.5], [0.0, 2.0, 1.0]])
    _, _, margin = oracle.geqrf(A[None])
    assert margin[0, 0] == 0.0 and margin[0, 1] > 1e-2
    R_ok, t_ok = _householder_sign_rule(A, flip=False)
    # flip only the first reflector (the tie): consistent QR, accepted
    alpha, x = A[0, 0], A[1:, 0]
    nu = np.linalg.norm(A[:, 0])
    beta = +nu
    tau0 = (beta - alpha) / beta
    v = np.concatenate([[1.0], x / (alpha - beta)])
    B = A.copy()
    B[1:, 0] = v[1:]
    B[0, 0] = beta
    C = B[:, 1:]
    C -= tau0 * np.outer(v, v @ C)
    Rt, tt = _householder_sign_rule(B[1:, 1:], flip=False)
    B[1:, 1:] = Rt
    taus = np.array([tau0, *tt])
    rep = compare_geqrf(oracle.to_cm(A[None].astype(np.float32)), 3, oracle.to_cm(B[None].astype(np.float32)),
                        taus[None].astype(np.float32))
    assert rep["ok"] and rep["flips"] >= 1 and rep["bad_flips"] == 0, rep
